# free-before-post (executors) and two-pixel Mandelbrot: tests, then A/B
F=gpurun_out/r3b; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh nfp "-DPAGODA_FREE_BEFORE_POST=0" nmp "-DPAGODA_MB_PAIR=0" > $F/variants.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py tests/test_cpp_api.py -q -x > $F/pytest_rt.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "mandelbrot or mm or mix" > $F/pytest_par.log 2>&1
for i in 1 2; do for v in 0 nfp nmp; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  if [ $v != nmp ]; then
  timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_$v\_$i.json
  timeout 200 python bench.py --workload mm --quick --no-configs --prespawn 2>/dev/null | tail -1 > $F/mmpre_$v\_$i.json
  timeout 200 python bench.py --workload nop --quick --no-configs 2>/dev/null | tail -1 > $F/nop_$v\_$i.json
  timeout 200 python bench.py --workload tdes --quick --no-configs 2>/dev/null | tail -1 > $F/tdes_$v\_$i.json
  timeout 200 python bench.py --workload mix --quick --no-configs 2>/dev/null | tail -1 > $F/mix_$v\_$i.json
  fi
  timeout 200 python bench.py --workload mb --quick --no-configs 2>/dev/null | tail -1 > $F/mb_$v\_$i.json
  timeout 200 python bench.py --workload mb --quick --no-configs --max-tasks 4 2>/dev/null | tail -1 > $F/mbm4_$v\_$i.json
done; done
unset PAGODA_LIB
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt; tail -3 $F/pytest_rt.log; tail -3 $F/pytest_par.log
