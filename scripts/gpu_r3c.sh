# CTA-scope executor fences with free-before-post; ingest timers compiled out
F=gpurun_out/r3c; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh cta "-DPAGODA_CTA_FENCE=1" nt "-DPAGODA_INGEST_TIMERS=0" ctant "-DPAGODA_CTA_FENCE=1 -DPAGODA_INGEST_TIMERS=0" > $F/variants.log 2>&1
export PAGODA_LIB=$PWD/build/variants/libpagoda_vctant.so
timeout 1200 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py -q -x > $F/pytest_ctant.log 2>&1
unset PAGODA_LIB
for i in 1 2; do for v in 0 cta nt ctant; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/mmpre_$v\_$i.json
  timeout 200 python bench.py --workload nop --quick --no-configs 2>/dev/null | tail -1 > $F/nop_$v\_$i.json
  timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
  timeout 200 python bench.py --workload mix --quick --no-configs 2>/dev/null | tail -1 > $F/mix_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt; tail -3 $F/pytest_ctant.log
