# ingest capacity (4 publishers) x MM / NOP; MB claim caps at 1 and 2 MTBs/SM; CONV shared-memory bands
F=gpurun_out/r2v; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh pub4 "-DPAGODA_INGEST_PUBLISHERS=4" > $F/variants.log 2>&1
timeout 600 python -m pytest tests/test_gpu_workloads.py -q -x -k "conv" > $F/pytest_conv.log 2>&1
for i in 1 2; do for v in 0 pub4; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/mmpre_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --mtbs 2 --groups 2 --arena-kb 64 2>/dev/null | tail -1 > $F/mm2g2_$v\_$i.json
done; done
unset PAGODA_LIB
for i in 1 2; do
  timeout 200 python bench.py --workload mix --quick --no-configs 2>/dev/null | tail -1 > $F/mix_0_$i.json
  for mt in 1 2 3; do timeout 200 python bench.py --workload mb --quick --no-configs --max-tasks $mt --spread 0 2>/dev/null | tail -1 > $F/mb_m${mt}_$i.json; done
  for mt in 1 2; do timeout 200 python bench.py --workload mb --quick --no-configs --max-tasks $mt --spread 0 --mtbs 2 --arena-kb 40 2>/dev/null | tail -1 > $F/mb_M2m${mt}_$i.json; done
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt; tail -2 $F/pytest_conv.log
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r2v/mm*_1.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, round(d["value"]/1e6,2), {k: round(v,3) for k,v in d["runtime_counters_per_task"].items()})
    except Exception as e: print(f, e)
PY
