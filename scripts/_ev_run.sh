OUT=final_r2b bash scripts/gpu_evidence.sh
