OUT=final_r2c bash scripts/gpu_evidence.sh
