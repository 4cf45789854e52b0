"""Build a compile-time variant of the library for an A/B measurement:
    python tools/ab_build.py /tmp/variant.so HISQ_ZT_NO_L1=0 [MORE=1 ...]
then run with HISQ_DSLASH_LIB=/tmp/variant.so (tests, bench.py) to load it instead of the default."""
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                "paper_conf_sc_dufekgaad024_b200"))
import build  # noqa: E402

print(build.build(force=True, defines=sys.argv[2:], out=os.path.abspath(sys.argv[1])))
