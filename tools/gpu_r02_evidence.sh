#!/bin/bash
# GPU-box helper (round 2 final evidence): GPU tests (incl. the full-size digest test), smoke, bench lines
# for every config (+ HashCube, k3_warps=24 and the reference arm at H), the ncu launch list of the default
# bench and one --set full capture of K3 at H (kept: tools/evidence_summary.py + traffic.json need it).
mkdir -p gpurun_out
rm -f gpurun_out/ev_*
python -c "from paper_conf_sigmod_boghcsa17_b200 import build; build.build()" || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/ev_gpu.txt
if [ "${TESTS:-1}" = 1 ]; then
  timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -6 > gpurun_out/ev_tests.log
fi
python __graft_entry__.py smoke > gpurun_out/ev_smoke.log 2>&1
for c in ${CONFIGS:-H C3A C3I C3C C2 C5 C4}; do
  timeout 900 python bench.py --config $c --cpu-seconds ${CPU_S:-8} 2>/dev/null | tail -1 > gpurun_out/ev_bench_$c.json
done
timeout 600 python bench.py --output hashcube --cpu-seconds 2 2>/dev/null | tail -1 > gpurun_out/ev_bench_H_hashcube.json
SKYCUBE_K3_WARPS=24 timeout 600 python bench.py --cpu-seconds 2 --no-e2e 2>/dev/null | tail -1 > gpurun_out/ev_bench_H_warps24.json
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 2>/dev/null | tail -1 > gpurun_out/ev_bench_H_reference.json
# ncu: the launch list of the default bench, then --set full captures of K3 (H, C4) and K1 (H); gpurun copies back
# at most 64 MiB, so every capture is summarised here (raw counters, per-source-line instructions and stall
# samples) and only the H K3 report is kept
summ() {
  ncu -i gpurun_out/$1.ncu-rep --page raw --csv > gpurun_out/$1.raw.csv 2>/dev/null
  python tools/ncu_lines.py gpurun_out/$1.ncu-rep 60 > gpurun_out/$1.lines.txt 2>/dev/null
  [ "$2" = keep ] || rm -f gpurun_out/$1.ncu-rep
}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches_H.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ev_ncu_launch.log 2>&1
if [ "${NCU_K3:-1}" = 1 ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k3_ -c 1 -f -o gpurun_out/ev_prof_k3_H \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config H > gpurun_out/ev_ncu_k3_H.log 2>&1
summ ev_prof_k3_H keep
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k3_ -c 1 -f -o gpurun_out/ev_prof_k3_C4 \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config C4 > gpurun_out/ev_ncu_k3_C4.log 2>&1
summ ev_prof_k3_C4
fi
# per-rank K1 / K3 work of an N-GPU run, measured on this one GPU (tools/k3_shard_time.py)
for c in ${SHARD_CONFIGS:-H C4}; do for w in 1 2 4 8; do timeout 900 python tools/k3_shard_time.py $c $w 3; done; done \
  > gpurun_out/ev_shards.jsonl 2> gpurun_out/ev_shards.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k1_prefilter -c 1 -f -o gpurun_out/ev_prof_k1_H \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config H > gpurun_out/ev_ncu_k1_H.log 2>&1
summ ev_prof_k1_H
cat gpurun_out/ev_tests.log gpurun_out/ev_smoke.log
for f in gpurun_out/ev_bench_*.json; do echo "$f: $(head -c 160 $f)"; done
du -sh gpurun_out
