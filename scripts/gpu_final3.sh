# Last measurement of the round with the final binary: smoke, GPU suite, every bench line, ncu full
# captures of the MasterKernel for 3DES, MM, the mix and NOP (runtime-only issue slots), launch list.
set -x
F=gpurun_out/final3; mkdir -p $F
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $F/smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $F/pytest_gpu.log 2>&1
timeout 900 python bench.py > $F/bench_tdes.json 2> $F/bench_tdes.err
for w in mb mm mm_tc mix c5 mpe tdes_var nop; do
  timeout 900 python bench.py --workload $w > $F/bench_$w.json 2> $F/bench_$w.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $F/launches_tdes.csv \
  python bench.py --prespawn --steps 3 --warmup 3 --no-naive --no-cpu --quick > $F/ncu_launch.log 2>&1
for w in tdes mm mix; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:master -s 3 -c 1 -o $F/${w}_full \
    python bench.py --workload $w --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > $F/${w}_full.log 2>&1
  python scripts/ncu_summary.py $F/${w}_full.ncu-rep > $F/ncu_${w}_full.txt 2>&1
done
timeout 900 ncu --set full --clock-control none -k regex:master -c 1 -o $F/nop_full python scripts/probe_runtime.py --ncu > $F/nop_full.log 2>&1
python scripts/ncu_summary.py $F/nop_full.ncu-rep > $F/ncu_nop_full.txt 2>&1
rm -f $F/*.ncu-rep
timeout 600 python scripts/probe_life.py nop mm tdes mix mb c5 mpe > $F/life.jsonl 2> $F/life.err
timeout 600 python scripts/probe_busy.py mm tdes nop mb > $F/busy.jsonl 2>&1
ls -la $F
