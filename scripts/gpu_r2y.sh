# 3DES rotated-domain rounds + full FMA-pipe sum: parity, then A/B
F=gpurun_out/r2y; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh nrot "-DPAGODA_TDES_ROT=0" nfs "-DPAGODA_TDES_FULL_SUM=0" old "-DPAGODA_TDES_ROT=0 -DPAGODA_TDES_FULL_SUM=0" > $F/variants.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_workloads.py -q -x -k "tdes or mpe or conv or c5" > $F/pytest.log 2>&1
for i in 1 2 3; do for v in 0 nrot nfs old; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
done; done
unset PAGODA_LIB
for i in 1 2; do timeout 200 python bench.py --workload mix --quick --no-configs 2>/dev/null | tail -1 > $F/mix_0_$i.json; done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt; tail -3 $F/pytest.log
