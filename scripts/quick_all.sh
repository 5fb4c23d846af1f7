# quick per-workload bench lines -> gpurun_out/q_<w>.json
for w in ${WORKLOADS:-tdes mb mm nop mix}; do
  timeout 300 python bench.py --workload $w --quick --no-cpu --no-naive 2>/dev/null | tail -1 > gpurun_out/q_$w.json
done
