"""Build a library variant (extra -D flags) into ab/ without touching the default library.
    python tools/variant.py prof -DGANNS_PROFILE=1            # d <= 128 instances only
    python tools/variant.py --full wide -DGANNS_WIDE_HINT=1   # every instance"""
import importlib.util
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
spec = importlib.util.spec_from_file_location("_b", os.path.join(ROOT, "paper_conf_icde_yuwzqzl22_b200", "_build.py"))
b = importlib.util.module_from_spec(spec)
spec.loader.exec_module(b)
args = sys.argv[1:]
full = "--full" in args
args = [a for a in args if a != "--full"]
name, defs = args[0], args[1:]
print(b.build_variant(os.path.join(ROOT, "ab", f"libganns_{name}.so"), defs, dev=not full))
