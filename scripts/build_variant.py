"""Build an experiment variant of libpt.so with -D overrides (same sources, same flags):
    python scripts/build_variant.py NAME -DPT_REFILL_MIN=4 ...  ->  scripts/libpt_NAME.so
Run it with PT_LIB=scripts/libpt_NAME.so (scripts/gpu.sh ab)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
name, defs = sys.argv[1], sys.argv[2:]
os.environ["PT_LIB"] = os.path.join(ROOT, "scripts", f"libpt_{name}.so")
os.environ["PT_NVCC_EXTRA"] = " ".join(defs)
sys.path.insert(0, ROOT)
from paper_conf_ipps_xuzwrwxgxy12_b200 import _build  # noqa: E402

print(_build.build(force=True))
