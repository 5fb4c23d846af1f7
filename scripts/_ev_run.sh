OUT=final_r2h bash scripts/gpu_evidence.sh
