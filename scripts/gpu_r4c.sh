# parallel validation for large single-producer spawns (npv = off)
F=gpurun_out/r4c; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh npv "-DPAGODA_PAR_VALIDATE_MIN=2000000000" > $F/variants.log 2>&1
timeout 900 python -m pytest tests/test_gpu_runtime.py -q -x > $F/pytest.log 2>&1; tail -2 $F/pytest.log
for i in 1 2 3; do for v in 0 npv; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
  timeout 200 python bench.py --workload mm_tc --quick --no-configs --producers 1 2>/dev/null | tail -1 > $F/mmtc1_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
