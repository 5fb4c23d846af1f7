OUT=final_r2g bash scripts/gpu_evidence.sh
