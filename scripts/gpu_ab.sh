# A/B of library variants (VARS="0 name ..." AB=outdir): parity subset, quick bench of every workload x2, lifecycle probe.
O=gpurun_out/${AB:-ab17}; mkdir -p $O
for v in ${VARS}; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 400 python -m pytest tests/test_gpu_parity.py tests/test_gpu_runtime.py -q -x -k "not full_size" 2>&1 | tail -1 > $O/t_$v.txt
  for w in nop mm tdes mb mix c5; do for i in 1 2; do
    timeout 300 python bench.py --workload $w --quick 2>/dev/null | tail -1 > $O/${w}_${v}_$i.json
  done; done
  timeout 300 python scripts/probe_life.py nop mm > $O/life_$v.jsonl 2>&1
done
python scripts/ab_summary.py $O
for v in ${VARS}; do python - $O/life_$v.jsonl <<'P'
import json, sys
for l in open(sys.argv[1]):
    try: d = json.loads(l)
    except Exception: continue
    print(sys.argv[1].split('/')[-1], d["workload"], round(d["tasks_per_s"]/1e6,1), {k: (round(v["mean_us"],1), round(v["in_stage"])) for k, v in d["stages"].items()})
P
done
