set -x
python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_tdes.csv python bench.py --prespawn --steps 3 --warmup 3 --no-naive --no-cpu --quick > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master -s 3 -c 1 -o gpurun_out/tdes_full python bench.py --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > gpurun_out/ncu_full_tdes.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master -s 3 -c 1 -o gpurun_out/mm_full python bench.py --workload mm --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > gpurun_out/ncu_full_mm.log 2>&1
ls -la gpurun_out
