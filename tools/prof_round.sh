#!/bin/bash
# One `ncu --set full` capture of a warm launch per workload (every kernel of
# that launch), for profiles/: run on the GPU box, then summarise here with
#   python tools/ncu_summary.py full gpurun_out/ncu_<W>_<TAG>.ncu-rep profiles/ncu_<W>_<TAG>.txt <W>
#   python tools/ncu_summary.py counters gpurun_out/ncu_<W>_<TAG>.ncu-rep <W>
# usage: bash tools/prof_round.sh <TAG> <workload> [...]   (never under a multi-rank command)
TAG=$1
shift
mkdir -p gpurun_out
for W in "$@"; do
  K=$(python tools/prof_workload.py "$W" 0 2>/dev/null | sed -n 's/.*kernels\/launch=\([0-9]*\).*/\1/p')
  echo "$W: $K kernels per launch"
  timeout 1200 ncu --set full --import-source on --clock-control none -k 'regex:ens_kernel|xs_items|xs_init_items|rs_items' \
    --launch-skip "$K" --launch-count "$K" -f -o "gpurun_out/ncu_${W}_${TAG}" \
    python tools/prof_workload.py "$W" 1 > "gpurun_out/ncu_${W}_${TAG}.log" 2>&1
  tail -1 "gpurun_out/ncu_${W}_${TAG}.log"
done
# summaries on the box (the reports exceed gpurun's 64 MiB copy-back): with
# SUMMARISE=1, gpurun_out/ gets the per-workload .txt, ncu_counters.json and
# traffic.json (copies of profiles/ updated), and the reports are removed
if [ "${SUMMARISE:-0}" = 1 ]; then
  cp profiles/ncu_counters.json gpurun_out/ncu_counters.json
  cp profiles/traffic.json gpurun_out/traffic.json
  for W in "$@"; do
    NCU_TRAFFIC=gpurun_out/traffic.json python tools/ncu_summary.py full "gpurun_out/ncu_${W}_${TAG}.ncu-rep" "gpurun_out/ncu_${W}_${TAG}.txt" "$W"
    NCU_COUNTERS=gpurun_out/ncu_counters.json python tools/ncu_summary.py counters "gpurun_out/ncu_${W}_${TAG}.ncu-rep" "$W"
    rm -f "gpurun_out/ncu_${W}_${TAG}.ncu-rep"
  done
fi
