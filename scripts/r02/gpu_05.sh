# round 2, call 5: copy progress under full SMs (probe v2); GEMM v2 debug
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/ce_probe scripts/ce_probe.cu -lcuda > /dev/null 2>&1 && timeout 60 /tmp/ce_probe
timeout 600 python scripts/gemm_debug.py 256x256x512 256x256x1024 256x512x2048 384x512x4096 2048x2048x16384 16384x16384x16384
