#!/bin/bash
# Per-rank ncu wrapper for multi-GPU runs (torchrun --no-python ... scripts/ncu_rank.sh <script> <args>):
# every rank's transfer kernels (send / relay / recv) are profiled in its own process with
# the NVLink, PCIe and DRAM byte counters and the launch duration, one CSV per rank.
# Only counters that ncu collects in a single pass are requested, so no kernel is
# replayed (a replayed send or relay kernel would re-run a handoff the peers already
# consumed).  Output: $NCU_OUT/ncu_rank<R>.csv (default gpurun_out/ncu_world).
OUT=${NCU_OUT:-gpurun_out/ncu_world}
mkdir -p "$OUT"
exec ncu --metrics gpu__time_duration.sum,nvltx__bytes_data_user.sum,nvlrx__bytes_data_user.sum,pcie__read_bytes.sum,pcie__write_bytes.sum \
  --clock-control none -k regex:"send_kernel|relay_kernel|recv_kernel" --csv \
  --log-file "$OUT/ncu_rank${RANK:-0}.csv" python "$@"
