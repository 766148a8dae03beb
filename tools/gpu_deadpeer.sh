#!/bin/bash
# Diagnose the dead-peer path: rank 1 skips its GEMM; rank 0 should fail after NORTHUP_PEER_TIMEOUT_S.
mkdir -p gpurun_out; python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
D=$(mktemp -d)
export PEER_SKIP_GEMM=1 NORTHUP_PEER_TIMEOUT_S=5 NORTHUP_DEBUG_EXEC=1
(timeout 40 python tests/peer_sibling.py $D 0 2 512 512 1024 256 0 int 1 > gpurun_out/dp0.log 2>&1; echo "rank0 rc=$?" >> gpurun_out/dp0.log) &
(timeout 50 python tests/peer_sibling.py $D 1 2 512 512 1024 256 0 int 1 > gpurun_out/dp1.log 2>&1; echo "rank1 rc=$?" >> gpurun_out/dp1.log) &
for i in $(seq 1 10); do sleep 5; echo "t=$((i*5)) files: $(ls $D | tr '\n' ' ')"; done
wait
head -30 gpurun_out/dp0.log; tail -8 gpurun_out/dp0.log; tail -5 gpurun_out/dp1.log
