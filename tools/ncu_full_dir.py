"""Summarise every .ncu-rep of a directory (key counters + top stalls per kernel) into one JSON (test-side)."""
import glob, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import summarize_full
src, out = sys.argv[1], sys.argv[2]
res = {os.path.basename(p)[:-8]: summarize_full(p) for p in sorted(glob.glob(os.path.join(src, "*.ncu-rep")))}
json.dump(res, open(out, "w"), indent=1)
print(out, list(res))
