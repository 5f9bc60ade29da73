#!/bin/bash
# Fused peer-memory exchange: chunk size x arrival signalling sweep (single rank and N virtual ranks),
# parity of the new variants, and a probe whether two NCCL ranks may share one GPU.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 120 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29611 \
    scripts/probe_nccl_dup.py > gpurun_out/nccl_dup.log 2>&1; echo "rc=$?" >> gpurun_out/nccl_dup.log
for sig in 1 0; do
  for ch in 2048 8192; do
    AVGPIPE_EA_P2P_SIGNAL=$sig AVGPIPE_EA_P2P_CHUNK=$ch timeout 900 python -m pytest tests/test_gpu_p2p.py -q -x > gpurun_out/pytest_p2p_s${sig}_c${ch}.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_p2p_s${sig}_c${ch}.log
  done
done
: > gpurun_out/p2p_sig.jsonl
for c in C4 C3N4; do
  for sig in 0 1; do
    for ch in 2048 4096 8192 16384; do
      for n in 1 0; do
        nn=""; [ $n = 1 ] && nn="--n 1"
        AVGPIPE_EA_P2P_SIGNAL=$sig AVGPIPE_EA_P2P_CHUNK=$ch timeout 200 python scripts/bench_p2p_virtual.py --config $c $nn \
          | sed "s/^{/{\"sig\": $sig, \"chunk\": $ch, /" >> gpurun_out/p2p_sig.jsonl 2>> gpurun_out/p2p_sig.err
      done
    done
  done
done
echo done
