#!/bin/bash
# GPU-box helper: tests, smoke, bench lines for every config, and the ncu launch list of the default bench.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m pytest tests -m gpu -x -q 2>&1 | tail -15
python __graft_entry__.py smoke
for c in ${CONFIGS:-H C4 C5 C3A C3I C2}; do
  timeout 600 python bench.py --steps 3 --warmup 3 --config $c --cpu-seconds ${CPU_S:-5} 2>gpurun_out/bench_$c.err | tail -1 > gpurun_out/bench_$c.json
  cat gpurun_out/bench_$c.json; tail -3 gpurun_out/bench_$c.err
done
if [ -z "$NO_NCU" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_h.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_b.log 2>&1
fi
