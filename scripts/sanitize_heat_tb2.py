"""heat3d_tb2 alone (P = 2 virtual partitions, ragged sizes) for compute-sanitizer racecheck /
synccheck: the shared exchange buffer of sweep-1 rows and its named barrier.

    compute-sanitizer --tool racecheck python scripts/sanitize_heat_tb2.py
"""
import sys

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import abi  # noqa: E402
from paper_conf_icppw_matzdf20_b200 import kernels as K  # noqa: E402


def main():
    ctx = abi.pk_init(2, part_device=[0, 0])
    h = synth.heat_grid(21, 37, 260)
    ph = K.heat3d_setup(ctx, h, zc=8, kernel="heat3d_tb2")
    K.heat3d_iterate(ph, 4)
    abi.pk_synchronize(ctx)
    abi.pk_finalize(ctx)
    print("heat3d_tb2 sanitize done")


if __name__ == "__main__":
    main()
