# round 2, call 6: GEMM v2 with the MN-major 128B_BASE32B layout
timeout 300 python scripts/gemm_debug.py 256x256x512 256x256x1024 256x512x2048 384x512x4096 2048x2048x16384
