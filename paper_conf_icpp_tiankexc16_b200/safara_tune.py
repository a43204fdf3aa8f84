"""SAFARA's static-feedback register assistant, applied to this kernel's
variant family.

The paper's loop (§III-B):
  1. classify every reused array reference by memory space and coalescing
     and count its uses (reference count C);
  2. compile without scalar replacement and read the hardware register count
     back from the assembler ("PTXAS Info", L764-786);
  3. cost each candidate L x C, L the access latency of its memory space,
     measured by microbenchmark (L823-835); sort;
  4. replace the most beneficial references with scalars while registers
     remain; recompile and go to 2 (L727-736).

`select()` is step 3-4 for one round; `feedback_loop()` iterates it against a
compile callback; the paper's running example (Fig. 5 -> Fig. 6:
26 registers used, limit 30 -> 4 free -> array b's 3 temporaries) is the unit
test.  `tune_variants()` applies the same idea to the hand-written kernel's
compile-time variant family: compile each variant, read registers / spill
bytes from ptxas, drop variants that spill or exceed the per-thread budget of
their CTA shape (the paper's "no register spilling" rule, L933-938), rank the
rest by a cost model built from the same latency table, and (optionally, on
a GPU) time the leaders with bench.py.

This is a build-time tool: it never runs on the hot path and never touches
the oracle.
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import dataclasses
import json
import os
import re
import subprocess
import sys
import tempfile

# Access latencies in SM cycles (B200/B300 microbenchmarks,
# /opt/skills/guides/B300_MICROARCH.md: L1 hit 32, L2 hit 234-262, DRAM ~580,
# LDS 29).  An uncoalesced warp access touches up to 32 sectors instead of the
# 8 of a coalesced fp64 row, so it costs ~4x the transactions.
LATENCY = {
    "register": 0,
    "shared": 29,
    "l1": 32,
    "global_coalesced": 250,
    "global_uncoalesced": 4 * 250,
    "dram": 580,
}


@dataclasses.dataclass(frozen=True)
class Candidate:
    """A group of reused array references SAFARA may turn into scalars.

    uses:  reference count C (reads + writes of the group in the loop body);
    space: memory space / access class (a key of LATENCY);
    regs:  temporaries (registers) the replacement needs."""
    name: str
    uses: int
    space: str
    regs: int

    def cost(self, latency: dict = LATENCY) -> int:
        return latency[self.space] * self.uses


def select(cands, used: int, limit: int, latency: dict = LATENCY):
    """One SAFARA round: free = limit - used registers; take candidates in
    decreasing L x C order while their temporaries fit.  Returns (chosen,
    free registers left)."""
    free = limit - used
    chosen = []
    for c in sorted(cands, key=lambda c: (-c.cost(latency), -c.uses, c.name)):
        if c.regs <= free and c.cost(latency) > 0:
            chosen.append(c)
            free -= c.regs
    return chosen, free


def feedback_loop(cands, compile_regs, limit: int, latency: dict = LATENCY, max_iter: int = 8):
    """Iterate compile -> registers -> select until no candidate fits.

    compile_regs(selected_names) -> registers used by the kernel compiled with
    those references replaced.  Returns (selected candidates, history of
    (iteration, selected names, registers))."""
    selected: list[Candidate] = []
    history = []
    for it in range(max_iter):
        regs = compile_regs(tuple(c.name for c in selected))
        history.append((it, tuple(c.name for c in selected), regs))
        rest = [c for c in cands if c not in selected]
        add, _ = select(rest, regs, limit, latency)
        if not add:
            break
        selected.extend(add[:1])  # one group per round, as the paper iterates
    return selected, history


# ---------------------------------------------------------------------------
# ptxas feedback ("PTXAS Info")
# ---------------------------------------------------------------------------
_FN = re.compile(r"Compiling entry function '([^']+)'")
_SPILL = re.compile(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads")
_REGS = re.compile(r"Used (\d+) registers")


def ptxas_info(log: str) -> dict:
    """{kernel: {"regs": r, "spill_st": s, "spill_ld": l, "stack": f}} from
    `nvcc -Xptxas -v` output."""
    out, cur = {}, None
    for line in log.splitlines():
        m = _FN.search(line)
        if m:
            cur = m.group(1)
            out[cur] = {"regs": None, "spill_st": 0, "spill_ld": 0, "stack": 0}
            continue
        if cur is None:
            continue
        m = _SPILL.search(line)
        if m:
            out[cur].update(stack=int(m.group(1)), spill_st=int(m.group(2)),
                            spill_ld=int(m.group(3)))
        m = _REGS.search(line)
        if m:
            out[cur]["regs"] = int(m.group(1))
    return out


# ---------------------------------------------------------------------------
# The kernel's variant family
# ---------------------------------------------------------------------------
@dataclasses.dataclass(frozen=True)
class Variant:
    ty: int = 12      # CTA tile rows (threads = 32*ty)
    stages: int = 4   # TMA ring depth
    rcp: int = 2      # reciprocal refinement (0: 3 Newton, 1: 2 Newton, 2: cubic)

    @property
    def threads(self) -> int:
        return 32 * self.ty

    @property
    def reg_limit(self) -> int:
        # one CTA per SM (shared memory); 64K registers, allocation granule 8
        return min(255, (65536 // self.threads) // 8 * 8)

    def defines(self) -> list[str]:
        return [f"-DSAFARA_TY={self.ty}", f"-DSAFARA_STAGES={self.stages}",
                f"-DSAFARA_RCP={self.rcp}"]

    def tag(self) -> str:
        return f"ty{self.ty}_s{self.stages}_r{self.rcp}"


def default_family() -> list[Variant]:
    return [Variant(ty, st, rcp) for ty in (8, 10, 12) for st in (3, 4) for rcp in (0, 2)]


def compile_variant(v: Variant, workdir: str) -> dict:
    """nvcc the production TU with the variant's defines; ptxas feedback."""
    from . import build as b
    cmd = [b.NVCC, *b.COMMON, "--fmad=true", "-Xptxas", "-v", *v.defines(), "-c",
           os.path.join(b.CSRC, "rhs_fast.cu"), "-o", os.path.join(workdir, v.tag() + ".o")]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        return {"variant": v, "error": res.stderr[-400:]}
    info = ptxas_info(res.stdout + res.stderr)
    prod = next((k for k in info if k.endswith("rhs_kernel_fast_udE14CUtensorMap_stS0_NS_6ParamsE")),
                None)
    return {"variant": v, "kernels": info, "prod": info.get(prod)}


def model_cost(v: Variant, regs: int) -> float:
    """Relative cycles per grid point of a variant (smaller is better), from
    the same latency table: the u tile's halo is re-read through L2
    ((32+6)(ty+4)/(32 ty) per point), latency hidden by the warps resident
    per SM scheduler (ty/4) and by the ring (stages-2 planes in flight)."""
    halo = (32 + 6) * (v.ty + 4) / (32 * v.ty)
    hide = (v.ty / 4) * max(1, v.stages - 2)
    rcp_fp64 = {0: 6, 1: 4, 2: 3}[v.rcp] * 4  # four reciprocals per point
    return halo * LATENCY["global_coalesced"] / hide + rcp_fp64 + 300


def tune_variants(family=None, jobs: int = 4) -> list[dict]:
    """Compile the family, apply SAFARA's feasibility rule (no spills, within
    the register budget of the CTA shape) and rank the survivors."""
    family = family or default_family()
    with tempfile.TemporaryDirectory() as wd:
        with cf.ThreadPoolExecutor(jobs) as ex:
            res = list(ex.map(lambda v: compile_variant(v, wd), family))
    rows = []
    for r in res:
        v, p = r["variant"], r.get("prod")
        if p is None:
            rows.append({"variant": v.tag(), "error": r.get("error", "no kernel")})
            continue
        ok = p["spill_st"] == 0 and p["spill_ld"] == 0 and p["regs"] <= v.reg_limit
        rows.append({"variant": v.tag(), "defines": v.defines(), "regs": p["regs"],
                     "reg_limit": v.reg_limit, "spill_bytes": p["spill_st"] + p["spill_ld"],
                     "feasible": ok, "model": round(model_cost(v, p["regs"]), 1)})
    rows.sort(key=lambda r: (not r.get("feasible", False), r.get("model", 1e9)))
    return rows


def time_variant(tag_defines, steps: int = 100) -> float | None:
    """Build the full library for a variant and time it with bench.py (GPU)."""
    from . import build as b
    tag, defines = tag_defines
    out = os.path.join(b.ROOT, "build", f"libsafara_{tag}.so")
    b.build(force=True, extra=defines, out=out)
    env = dict(os.environ, SAFARA_LIB=out)
    res = subprocess.run([sys.executable, os.path.join(b.ROOT, "bench.py"), "--steps", str(steps),
                          "--warmup", "10", "--no-cpu-baseline", "--no-other-configs", "--soak-s", "0.3",
                          "--e2e-steps", "0"], capture_output=True, text=True, env=env)
    try:
        return json.loads(res.stdout.strip().splitlines()[-1])["roofline"]["kernel_ms"] * 1e3
    except Exception:
        return None


def main(argv=None):
    ap = argparse.ArgumentParser(description=__doc__.split("\n\n")[0])
    ap.add_argument("--time", type=int, default=0, help="time the N best feasible variants (GPU)")
    ap.add_argument("--jobs", type=int, default=4)
    a = ap.parse_args(argv)
    rows = tune_variants(jobs=a.jobs)
    for r in rows:
        print(json.dumps(r))
    if a.time:
        for r in [r for r in rows if r.get("feasible")][:a.time]:
            us = time_variant((r["variant"], r["defines"]))
            print(json.dumps({"variant": r["variant"], "kernel_us": us}))


if __name__ == "__main__":
    main()
