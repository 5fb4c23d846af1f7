F=gpurun_out/r2m; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh ws0 "-DPAGODA_WAIT_SLEEP_MAX=0" ws256 "-DPAGODA_WAIT_SLEEP_MAX=256" ws4k "-DPAGODA_WAIT_SLEEP_MAX=4096" nodi "-DPAGODA_DIRECT_IDLE_NS=0" > $F/variants.log 2>&1
timeout 900 python -m pytest tests/test_gpu_bruteforce.py tests/test_gpu_runtime.py -m gpu -q -x > $F/pytest.log 2>&1
VARS="0 ws0 ws256 ws4k nodi" AB=r2m ABW="tdes mm nop mb mix" bash scripts/gpu_ab.sh > $F/ab.txt 2>&1
timeout 300 python bench.py --no-configs --no-naive --no-cpu 2>/dev/null | tail -1 > $F/full.json
python -c "import json;d=json.loads(open('$F/full.json').read());print('full', round(d['value']/1e6,2), d['roofline']['frac'], 'e2e', round(d['e2e']['value']/1e6,2), 'iso', d['latency']['isolated_nop128_us']['p50'], d['latency']['isolated_nop128_over_floor'], 'p50', d['p50_spawn_to_done_us'])" >> $F/ab.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master_kernel -c 1 -o $F/ncu_tdes python bench.py --quick --no-configs --prespawn --steps 1 --warmup 0 > $F/ncu_run.log 2>&1
tail -3 $F/pytest.log; cat $F/ab.txt
