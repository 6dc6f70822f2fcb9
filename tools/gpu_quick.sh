#!/bin/bash
# GPU-box helper: GPU tests, then the H bench (and CONFIGS), then an ncu capture of K3 at H (NCU=1).
mkdir -p gpurun_out
python -c "from paper_conf_sigmod_boghcsa17_b200 import build; build.build()"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/q_tests.log
cat gpurun_out/q_tests.log
for c in ${CONFIGS:-H}; do
  timeout 600 python bench.py --steps 3 --warmup 3 --config $c --cpu-seconds ${CPU_S:-2} 2>gpurun_out/q_bench_$c.err | tail -1 > gpurun_out/q_bench_$c.json
  python tools/bench_summary.py gpurun_out/q_bench_$c.json 2>/dev/null || tail -c 600 gpurun_out/q_bench_$c.json
done
if [ -n "$NCU" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KERNEL:-k3_mdmc} -c 1 -f -o gpurun_out/q_prof \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config ${NCU_CFG:-H} > gpurun_out/q_ncu.log 2>&1
  tail -2 gpurun_out/q_ncu.log
fi
