# 3DES body as a call (default now; tin = inlined): other workloads, parity
F=gpurun_out/r4e; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh tin "-DPAGODA_TDES_NOINLINE=0" > $F/variants.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_workloads.py -q -x -k "tdes or mpe or c5" > $F/pytest.log 2>&1; tail -2 $F/pytest.log
for i in 1 2; do for v in 0 tin; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  for w in mm mb mix tdes_var mpe; do timeout 200 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $F/${w}_$v\_$i.json; done
  timeout 300 python bench.py --workload c5 --quick --no-configs --steps 3 --warmup 1 2>/dev/null | tail -1 > $F/c5_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
