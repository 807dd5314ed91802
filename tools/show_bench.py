"""Print selected keys of a bench.py JSON line:  python tools/show_bench.py <file> key [key ...]"""
import json
import sys

d = json.loads(open(sys.argv[1]).readline())
for k in sys.argv[2:]:
    v = d.get(k)
    print(k, v["value"] if isinstance(v, dict) and "value" in v else v)
