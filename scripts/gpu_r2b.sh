# round 2: pool tests, the default bench line (all five configs), pool bench at --gpus 2
F=gpurun_out/r2b; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_runtime.py -m gpu -q -x -k "pool or nonblocking or sync_without or paper or 255" > $F/pytest_pool.log 2>&1
timeout 1200 python bench.py > $F/bench_default.json 2> $F/bench_default.err
timeout 600 python bench.py --gpus 2 --workload c5 --steps 5 > $F/bench_pool_c5.json 2> $F/bench_pool_c5.err
timeout 600 python bench.py --gpus 2 --steps 10 > $F/bench_pool_tdes.json 2> $F/bench_pool_tdes.err
tail -3 $F/pytest_pool.log
