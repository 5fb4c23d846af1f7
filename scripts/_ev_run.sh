OUT=final_r2i bash scripts/gpu_evidence.sh
