# A/B of library variants: VARS="0 name ..." AB=outdir [ABW="mm nop tdes"] [TESTS=1] bash scripts/gpu_ab.sh
# (variants built by scripts/build_variants.sh; 0 = the in-tree build).  Per variant: optionally the
# runtime GPU tests, then a quick bench of every workload x2; summary by scripts/ab_summary.py.
O=gpurun_out/${AB:-ab}; mkdir -p $O
for v in ${VARS:-0}; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  if [ "${TESTS:-0}" = 1 ]; then
    timeout 600 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py tests/test_gpu_parity.py -m gpu -q -x -k "not full_size" 2>&1 | tail -2 > $O/t_$v.txt
  fi
  for w in ${ABW:-mm nop tdes mb mix}; do for i in 1 2; do
    timeout 300 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $O/${w}_${v}_$i.json
  done; done
done
python scripts/ab_summary.py $O
