#!/bin/bash
# Multi-rank engine, 2 ranks on one GPU under MPS: per-message time of back-to-back
# sends (scripts/diag_world_perf.py) with and without PDL.  Usage: bash scripts/world_pdl.sh <outdir>
OUT=${1:-gpurun_out/world_pdl}
mkdir -p $OUT
for pdl in 1 0; do
  for n in 65536 1048576 16777216; do
    MPX_PDL_WORLD=$pdl DIAG_BYTES=$n DIAG_K=200 MPX_BENCH_SAME_GPU=1 timeout 180 python -m torch.distributed.run \
      --standalone --local-addr 127.0.0.1 --nproc-per-node 2 scripts/diag_world_perf.py \
      > $OUT/pdl${pdl}_n${n}.jsonl 2> $OUT/pdl${pdl}_n${n}.err
    echo "pdl=$pdl n=$n rc=$?" >> $OUT/rc.txt
  done
done
