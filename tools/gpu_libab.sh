#!/bin/bash
# GPU-box helper: A/B of library builds (LIBS, in-tree .so names built with SKYCUBE_BUILD_SUFFIX and
# SKYCUBE_NVCC_EXTRA), bench lines for CONFIGS, then (TESTS=1) the GPU parity tests against each library.
mkdir -p gpurun_out
P=paper_conf_sigmod_boghcsa17_b200
for c in ${CONFIGS:-H}; do
  for l in ${LIBS:-libskycube.so}; do
    SKYCUBE_LIB=$PWD/$P/$l timeout 600 python bench.py --steps 3 --warmup 3 --config $c --no-e2e --no-cpu 2>/dev/null | tail -1 > gpurun_out/lab_${c}_$l.json
    python tools/bench_summary.py gpurun_out/lab_${c}_$l.json "$l"
  done
done
if [ "${TESTS:-0}" != 0 ]; then
  for l in ${LIBS:-libskycube.so}; do
    SKYCUBE_LIB=$PWD/$P/$l timeout 1200 python -m pytest tests -m gpu -x -q ${TEST_ARGS:-} 2>&1 | tail -3 > gpurun_out/lab_tests_$l.log
    echo "$l: $(tail -1 gpurun_out/lab_tests_$l.log)"
  done
fi
