# MM body: A rows as float4 (vec), as a call (noinline): parity, then A/B
F=gpurun_out/r3g; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh nv "-DPAGODA_MM_VEC=0" old "-DPAGODA_MM_VEC=0 -DPAGODA_MM_NOINLINE=0" > $F/variants.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_workloads.py -q -x -k "mm or mpe or c5 or chain" > $F/pytest.log 2>&1; tail -3 $F/pytest.log
for i in 1 2; do for v in 0 nv old; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/mmpre_$v\_$i.json
  timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
  timeout 300 python bench.py --workload c5 --quick --no-configs --steps 2 --warmup 1 2>/dev/null | tail -1 > $F/c5_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
for i in 1 2; do
  timeout 200 python bench.py --workload mix --quick --no-configs 2>/dev/null | tail -1 > $F/mix_m1_$i.json
  timeout 200 python bench.py --workload mix --quick --no-configs --mtbs 3 --arena-kb 64 2>/dev/null | tail -1 > $F/mix_m3_$i.json
  timeout 300 python bench.py --workload c5 --quick --no-configs --steps 2 --warmup 1 --mtbs 3 --arena-kb 64 --no-resident 2>/dev/null | tail -1 > $F/c5_m3nr_$i.json
  timeout 300 python bench.py --workload c5 --quick --no-configs --steps 2 --warmup 1 --no-resident 2>/dev/null | tail -1 > $F/c5_m1nr_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --mtbs 3 --arena-kb 48 2>/dev/null | tail -1 > $F/mm_m3_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --mtbs 3 --arena-kb 48 2>/dev/null | tail -1 > $F/mb_m3_$i.json
done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
