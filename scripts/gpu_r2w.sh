# CONV variants on mix (shared-memory bands / inlining) + 4 ingest publishers on MM
F=gpurun_out/r2w; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh pub4 "-DPAGODA_INGEST_PUBLISHERS=4" nb "-DPAGODA_CONV_MIN_BAND=100000" inl "-DPAGODA_CONV_INLINE=1" inlnb "-DPAGODA_CONV_INLINE=1 -DPAGODA_CONV_MIN_BAND=100000" > $F/variants.log 2>&1
for i in 1 2; do for v in 0 nb inl inlnb; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload mix --quick --no-configs 2>/dev/null | tail -1 > $F/mix_$v\_$i.json
done; done
for i in 1 2; do for v in 0 pub4; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/mmpre_$v\_$i.json
  timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r2w/mm*_1.json")+glob.glob("gpurun_out/r2w/tdes*_1.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, round(d["value"]/1e6,2), {k: round(v,3) for k,v in d["runtime_counters_per_task"].items()})
    except Exception as e: print(f, e)
PY
