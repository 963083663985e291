PK_NVCC_FLAGS="-DPK_HEATTB_V=2 -DPK_HEATTB_MINB=4" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
PK_HEATTB_COLS=60 timeout 300 compute-sanitizer --tool memcheck python scripts/heat_v2_probe.py 2>&1 | head -40
