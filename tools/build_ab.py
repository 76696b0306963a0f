"""Build libtbs.so variants under build/ab/ for on-GPU A/B runs (TBS_LIB_VARIANT=...)."""
import os
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icpp_pitaksirianannt16_b200 import build as b  # noqa: E402

VARIANTS = {}
for arg in sys.argv[1:]:               # name=DEF1+DEF2  (values may contain commas)
    name, defs = arg.split("=", 1)
    VARIANTS[name] = [d for d in defs.split("+") if d]

os.makedirs(os.path.join(ROOT, "build", "ab"), exist_ok=True)
with ThreadPoolExecutor(8) as ex:
    futs = {n: ex.submit(b.build, True, False, os.path.join(ROOT, "build", "ab", f"libtbs_{n}.so"), d)
            for n, d in VARIANTS.items()}
    for n, f in futs.items():
        print(n, f.result())
