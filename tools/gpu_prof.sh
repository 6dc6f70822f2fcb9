#!/bin/bash
# GPU-box helper: ncu launch list + one capture per kernel regex for a config (default H).
#   CFG=H KERNELS="k3_mdmc k1_prefilter" FULL=1 bash tools/gpu_prof.sh
C=${CFG:-H}
mkdir -p gpurun_out
python -c "from paper_conf_sigmod_boghcsa17_b200 import build; build.build()"
if [ -z "$NO_LAUNCH" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$C.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config $C > gpurun_out/ncu_launch_$C.log 2>&1
fi
if [ -n "$FULL" ]; then SEC="--set full"; else
SEC="--section SpeedOfLight --section LaunchStats --section Occupancy --section WarpStateStats --section SourceCounters --section InstructionStats --section ComputeWorkloadAnalysis --section MemoryWorkloadAnalysis --metrics sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,sm__issue_active.avg.pct_of_peak_sustained_active"; fi
for K in ${KERNELS:-k3_mdmc k1_prefilter}; do
timeout 1200 ncu $SEC --clock-control none --import-source on -k regex:$K -c 1 -f -o gpurun_out/prof_${K}_$C \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config $C > gpurun_out/ncu_${K}_$C.log 2>&1
tail -2 gpurun_out/ncu_${K}_$C.log
done
