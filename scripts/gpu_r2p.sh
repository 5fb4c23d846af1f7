F=gpurun_out/r2p; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh fg1 "-DPAGODA_FIXED_GROUPS=1" > $F/variants.log 2>&1
timeout 300 python -m pytest tests/test_gpu_runtime.py -m gpu -q -x -k lifecycle > $F/pytest.log 2>&1
for i in 1 2 3; do for v in 0 fg1; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  for pr in 1 2; do timeout 200 python bench.py --quick --no-configs --producers $pr 2>/dev/null | tail -1 > $F/tdes${pr}_${v}_$i.json; done
  timeout 200 python bench.py --quick --no-configs --workload mm 2>/dev/null | tail -1 > $F/mm_${v}_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt
tail -2 $F/pytest.log; cat $F/ab.txt
