"""Engine utilisation and idle gaps of a decision trace (any timing mode).

    python tools/trace_gaps.py trace.txt [--top 15]

For each (gid, engine, slot): busy time (START->DONE), idle time between its
first START and last DONE, the largest gaps and which phases were woken /
waiting at that moment.
"""
import sys
from collections import defaultdict


def load(path):
    recs = []
    for ln in open(path):
        f = ln.split()
        if len(f) == 10:
            recs.append(f)
    return recs


def main():
    path = sys.argv[1]
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 10
    recs = load(path)
    t0 = int(recs[0][0])
    t1 = int(recs[-1][0])
    busy = defaultdict(list)
    start = {}
    for f in recs:
        t, kind = int(f[0]), f[1]
        if kind == "START":
            start[(f[2], f[3], f[4], f[7])] = t
        elif kind == "DONE":
            s = start.pop((f[2], f[3], f[4], f[7]))
            busy[(f[2], f[3], f[4])].append((s, t, f[5], f[7]))
    span = (t1 - t0) / 1e6
    print(f"trace span {span:.3f} ms, {len(recs)} records")
    for key in sorted(busy):
        iv = sorted(busy[key])
        b = sum(e - s for s, e, _, _ in iv)
        first, last = iv[0][0], iv[-1][1]
        gaps = [(iv[i + 1][0] - iv[i][1], iv[i][1], iv[i + 1][0]) for i in range(len(iv) - 1)]
        gaps.sort(reverse=True)
        idle = sum(g for g, _, _ in gaps)
        print(f"gid {key[0]} {key[1]:>3} slot {key[2]}: ops {len(iv):4d} busy {b / 1e6:8.3f} ms "
              f"active window {(last - first) / 1e6:8.3f} ms idle {idle / 1e6:7.3f} ms "
              f"(lead {(first - t0) / 1e6:.3f}, tail {(t1 - last) / 1e6:.3f})")
        for g, a, bb in gaps[:top]:
            if g > 0:
                print(f"      gap {g / 1e3:9.1f} us at {(a - t0) / 1e6:8.3f} ms")


if __name__ == "__main__":
    main()
