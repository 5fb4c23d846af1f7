OUT=final_r2f bash scripts/gpu_evidence.sh
