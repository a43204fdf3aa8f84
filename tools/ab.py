"""A/B experiments on compile-time / environment variants of the library.

  python tools/ab.py build NAME=-DFLAG=1,-DOTHER=2 ...   (here, on CPU)
      builds ablibs/NAME.so with those extra nvcc flags (in parallel)
  python tools/ab.py run REPS SPEC ...                    (on the GPU box)
      SPEC = LIB[+ENV=V[+ENV=V]] with LIB a name built above or 'default';
      interleaved bench.py runs (BT class C, production), kernel time each,
      one JSON line per run and a summary (min / median per spec).
"""
import concurrent.futures as cf
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
ABLIBS = os.path.join(ROOT, "ablibs")


def build(specs):
    from paper_conf_icpp_tiankexc16_b200 import build as b
    os.makedirs(ABLIBS, exist_ok=True)

    def one(spec):
        name, _, flags = spec.partition("=")
        extra = [f for f in flags.split(",") if f]
        out = os.path.join(ABLIBS, name + ".so")
        b.build(force=True, extra=extra, out=out, objdir=os.path.join(ABLIBS, "obj_" + name))
        log = open(out + ".ptxas.txt").read()
        spills = [l.strip() for l in log.splitlines() if "spill" in l and not l.strip().startswith("0 bytes stack")]
        return name, extra, spills

    with cf.ThreadPoolExecutor(4) as ex:
        for name, extra, spills in ex.map(one, specs):
            print(f"built {name} {extra} spills: {spills[:4]}")


def run(reps, specs, steps=400):
    res = {s: [] for s in specs}
    for rep in range(reps):
        for spec in specs:
            lib, *envs = spec.split("+")
            env = dict(os.environ)
            if lib != "default":
                env["SAFARA_LIB"] = os.path.join(ABLIBS, lib + ".so")
            for e in envs:
                k, _, v = e.partition("=")
                env[k] = v
            r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", str(steps),
                                "--warmup", "20", "--no-cpu-baseline", "--no-other-configs", "--e2e-steps", "1"],
                               capture_output=True, text=True, env=env, timeout=600)
            try:
                d = json.loads(r.stdout.strip().splitlines()[-1])
                us = d["ms_per_step"] * 1e3
                line = {"spec": spec, "rep": rep, "us": round(us, 2),
                        "frac": round(d["roofline"]["frac"], 4), "sm_mhz": d["clocks"]["sm_mhz"]}
            except Exception:
                us, line = None, {"spec": spec, "rep": rep, "error": r.stderr[-300:]}
            res[spec].append(us)
            print(json.dumps(line), flush=True)
    for s, t in res.items():
        t = [x for x in t if x]
        if t:
            print(json.dumps({"spec": s, "min_us": round(min(t), 2),
                              "median_us": round(statistics.median(t), 2), "n": len(t)}))


if __name__ == "__main__":
    if sys.argv[1] == "build":
        build(sys.argv[2:])
    else:
        run(int(sys.argv[2]), sys.argv[3:])
