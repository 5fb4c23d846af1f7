F=gpurun_out/r2l; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh dp "-DPAGODA_DIRECT_POST=1" > $F/variants.log 2>&1
timeout 600 python -m pytest tests/test_gpu_bruteforce.py -m gpu -q -x > $F/pytest.log 2>&1
PAGODA_LIB=$PWD/build/variants/libpagoda_vdp.so timeout 600 python -m pytest tests/test_gpu_runtime.py -m gpu -q -x -k "nop_many or mark or sessions or ring_wrap or chain or lifecycle" > $F/pytest_dp.log 2>&1
VARS="0 dp" AB=r2l ABW="mm tdes nop mix" bash scripts/gpu_ab.sh > $F/ab.txt 2>&1
for v in 0 dp; do if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 300 python bench.py --no-configs --no-naive --no-cpu 2>/dev/null | tail -1 > $F/full_$v.json
  python -c "import json;d=json.loads(open('$F/full_$v.json').read());print('$v', round(d['value']/1e6,2), 'e2e', round(d['e2e']['value']/1e6,2), 'iso', d['latency']['isolated_nop128_us']['p50'], 'p50', d['p50_spawn_to_done_us'])" >> $F/ab.txt
done
tail -2 $F/pytest.log $F/pytest_dp.log; cat $F/ab.txt
