# MMA issue cost without pipeline drains (scripts/micro/mma_ring.cu)
cd $GRAFT_REPO_ROOT
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mma_ring scripts/micro/mma_ring.cu || exit 1
timeout 300 /tmp/mma_ring > gpurun_out/mma_ring.txt 2>&1; cat gpurun_out/mma_ring.txt
