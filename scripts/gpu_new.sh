# new workloads: parity tests + bench lines
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python -m pytest tests/test_gpu_workloads.py -x -q > gpurun_out/pytest_wl.log 2>&1; tail -3 gpurun_out/pytest_wl.log
for w in ${WORKLOADS:-c5 mpe tdes_var mix}; do
  timeout 600 python bench.py --workload $w --no-naive --no-e2e --steps 5 --warmup 3 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
  python -c "import json;d=json.loads(open('gpurun_out/bench_$w.json').read().strip().splitlines()[-1]);print('$w',d['value'],d['ms_per_step'],d['roofline']['resource'],d['roofline']['frac'],d.get('p50_spawn_to_done_us'))" || tail -5 gpurun_out/bench_$w.err
done
