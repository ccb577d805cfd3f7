# Final evidence run for this build: GPU tests, smoke, launch list + ncu of the
# SGEMM launch (summarised into profiles/ on the box, copied back through
# gpurun_out/), then the bench (which reads the fresh traffic stamp).
set -x
mkdir -p gpurun_out/final
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/final/gputest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" >> gpurun_out/final/gputest.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final/launches.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e --no-alt-mode --no-context --no-routine-clocks --no-fp64 \
  > gpurun_out/final/ncu_launch.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_structured -c 1 -o gpurun_out/final/sgemm \
  python tools/one_call.py sgemm 8192 > gpurun_out/final/ncu_sgemm.log 2>&1
python tools/ncu_summary.py r02 gpurun_out/final/launches.csv gpurun_out/final/sgemm.ncu-rep > gpurun_out/final/summary.log 2>&1
cp profiles/r02_launches.md profiles/r02_sgemm_ncu.md profiles/ncu_sgemm_traffic.json gpurun_out/final/
timeout 900 python bench.py > gpurun_out/final/bench.json 2> gpurun_out/final/bench.err
timeout 900 python bench.py --workload cfg5 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/final/cfg5.json 2> gpurun_out/final/cfg5.err
