set -e
mkdir -p /tmp/pb
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pb/ystore tools/ystore_bench.cu
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pb/xload tools/xload_bench.cu -lcuda
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pb/umma_rate tools/umma_rate.cu -lcuda || true
echo "== ystore"; timeout 60 /tmp/pb/ystore
echo "== xload"; timeout 60 /tmp/pb/xload
echo "== umma_rate"; timeout 60 /tmp/pb/umma_rate || true
