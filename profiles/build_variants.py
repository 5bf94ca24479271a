"""Build tuning variants of libigd into variants/ (git-ignored), e.g.
   python profiles/build_variants.py lb1:IGD_SORT_LB=1 lb8:IGD_SORT_LB=8,IGD_SORT_ITEMS=24"""
import os
import sys
from concurrent.futures import ThreadPoolExecutor

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sosp_kamathb21_b200 import _build  # noqa: E402

os.makedirs("variants", exist_ok=True)


def one(spec):
    name, _, defs = spec.partition(":")
    return _build.build(defines=[d for d in defs.split(",") if d], out=f"variants/libigd_{name}.so")


with ThreadPoolExecutor(8) as ex:
    for p in ex.map(one, sys.argv[1:]):
        print(p)
