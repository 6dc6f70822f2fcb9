#!/bin/bash
# GPU-box helper (round 2): build check, integer-peak microbenchmark, GPU tests (TESTS=0 skips; TESTK=expr
# selects), bench lines for CONFIGS, optional ncu capture of K3 (NCU=1, NCU_CFG=H).
mkdir -p gpurun_out
python -c "from paper_conf_sigmod_boghcsa17_b200 import build; build.build()" || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv,noheader > gpurun_out/r02_gpu.txt
if [ "${INTPEAK:-1}" = 1 ]; then
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/intpeak tools/intpeak.cu && \
    timeout 300 /tmp/intpeak > gpurun_out/r02_intpeak.json 2> gpurun_out/r02_intpeak.err
  cat gpurun_out/r02_intpeak.json
fi
if [ "${TESTS:-1}" = 1 ]; then
  timeout ${TEST_TIMEOUT:-1500} python -m pytest tests -m gpu -x -q ${TESTK:+-k "$TESTK"} > gpurun_out/r02_tests.log 2>&1
  tail -5 gpurun_out/r02_tests.log
fi
for c in ${CONFIGS:-H}; do
  timeout 900 python bench.py --steps ${STEPS:-5} --warmup 3 --config $c --cpu-seconds ${CPU_S:-2} ${BENCH_EXTRA} \
    2> gpurun_out/r02_bench_$c.err | tail -1 > gpurun_out/r02_bench_$c.json
  python tools/bench_summary.py gpurun_out/r02_bench_$c.json 2>/dev/null || tail -c 800 gpurun_out/r02_bench_$c.json
done
if [ -n "$NCU" ]; then
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:${KERNEL:-k3_} -c 1 -f \
    -o gpurun_out/r02_prof_${NCU_CFG:-H} \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config ${NCU_CFG:-H} > gpurun_out/r02_ncu.log 2>&1
  tail -2 gpurun_out/r02_ncu.log
fi
