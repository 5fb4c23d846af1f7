OUT=final_r2e bash scripts/gpu_evidence.sh
