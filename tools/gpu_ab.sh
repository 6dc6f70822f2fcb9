#!/bin/bash
# GPU-box helper: parity tests, then bench lines per config for each value of an env switch.
#   VAR=SKYCUBE_K3_SUPER VALUES="0 1" CONFIGS="H C5" bash tools/gpu_ab.sh
mkdir -p gpurun_out
python -c "from paper_conf_sigmod_boghcsa17_b200 import build; build.build()" || exit 1
if [ -z "$NO_TEST" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1
  tail -3 gpurun_out/pytest_gpu.log
fi
for c in ${CONFIGS:-H}; do
  for v in ${VALUES:-default}; do
    tag=$(basename "$v")
    if [ "$v" = default ]; then
      timeout 600 python bench.py --steps ${STEPS:-3} --warmup 3 --config $c --no-cpu --no-e2e 2>gpurun_out/ab_${c}_$tag.err | tail -1 > gpurun_out/ab_${c}_$tag.json
    else
      env $VAR=$v timeout 600 python bench.py --steps ${STEPS:-3} --warmup 3 --config $c --no-cpu --no-e2e 2>gpurun_out/ab_${c}_$tag.err | tail -1 > gpurun_out/ab_${c}_$tag.json
    fi
    python tools/bench_summary.py gpurun_out/ab_${c}_$tag.json "$c $VAR=$v"
  done
done
