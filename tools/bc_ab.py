"""In-process interleaved A/B of bulge-chase variants selected by environment (read by libtrid at every call):
  python tools/bc_ab.py N B REPS "name:VAR=val,VAR2=val" ...
Every variant runs on the same band (one seeded SBR), round-robin REPS times; prints the median per variant and
whether its outputs equal the first variant's bit for bit."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_wangdzwzljz25_b200 as trid  # noqa: E402
import trid_gen  # noqa: E402


def main():
    n, b, reps = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
    variants = []
    for spec in sys.argv[4:]:
        name, _, envs = spec.partition(":")
        env = dict(kv.split("=", 1) for kv in envs.split(",") if kv)
        variants.append((name, env))
    A = trid_gen.random_symmetric(n, 3001 if n >= 32768 else 2001, device="cuda")
    trid.sbr_dbbr(A, b, nb=min(16, b), k=1024)
    nbytes, _, _ = trid.bulge_chase_bufsize(n, b)
    work = torch.zeros(nbytes, dtype=torch.uint8, device="cuda")
    st = torch.cuda.current_stream()
    base = dict(os.environ)
    times = {name: [] for name, _ in variants}
    ref = None
    same = {}
    for r in range(reps + 1):
        for name, env in variants:
            os.environ.clear()
            os.environ.update(base)
            os.environ.update(env)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            out = trid.bulge_chase(A, b, work=work)
            e1.record(st)
            torch.cuda.synchronize()
            if r == 0:
                outs = [x.clone() for x in out]
                if ref is None:
                    ref = outs
                same[name] = all(torch.equal(x, y) for x, y in zip(ref, outs))
                continue
            times[name].append(e0.elapsed_time(e1))
    os.environ.clear()
    os.environ.update(base)
    for name, env in variants:
        ts = times[name]
        print(json.dumps({"n": n, "b": b, "variant": name, "env": env, "median_ms": round(statistics.median(ts), 3),
                          "min_ms": round(min(ts), 3), "max_ms": round(max(ts), 3), "bitwise_equal_first": same[name]}))


if __name__ == "__main__":
    main()
