# Round measurement: default bench line, ncu launch list (self-draining sessions, as ncu
# serialises launches), --set full captures of the MasterKernel (3DES, MM), PCIe contention probe.
set -x
python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_tdes.csv \
  python bench.py --prespawn --steps 3 --warmup 3 --no-naive --no-cpu --quick > gpurun_out/ncu_launch.log 2>&1
bash scripts/ncu_tdes.sh tdes_full tdes
bash scripts/ncu_tdes.sh mm_full mm
timeout 300 python scripts/probe_contention.py > gpurun_out/contention.json
for w in mb mm mix nop; do timeout 600 python bench.py --workload $w --no-cpu > gpurun_out/bench_$w.json 2>/dev/null; done
ls -la gpurun_out
