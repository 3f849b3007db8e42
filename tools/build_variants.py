"""Build tuning variants of libtempgraph.so into variants/ (git-ignored; they travel with gpurun)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import _build  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.makedirs(os.path.join(ROOT, "variants"), exist_ok=True)
for spec in sys.argv[1:]:  # name:FLAG=V,FLAG=V
    name, _, fl = spec.partition(":")
    flags = tuple("-D" + f for f in fl.split(",") if f)
    print(name, flags, _build.build(force=True, extra_flags=flags,
                                    out=os.path.join(ROOT, "variants", f"lib_{name}.so")), flush=True)
