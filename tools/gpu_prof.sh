#!/bin/bash
# GPU-box helper: ncu launch list + one --set full capture of K3 and K1 for a config (default H).
C=${CFG:-H}
mkdir -p gpurun_out
python -c "from paper_conf_sigmod_boghcsa17_b200 import build; build.build()"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$C.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config $C > gpurun_out/ncu_launch_$C.log 2>&1
for K in ${KERNELS:-k3_mdmc k1_prefilter}; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -c 1 -f -o gpurun_out/prof_${K}_$C \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config $C > gpurun_out/ncu_${K}_$C.log 2>&1
done
