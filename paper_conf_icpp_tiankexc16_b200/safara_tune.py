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

# Access latencies in SM cycles, measured on the B200 by the [19]-style
# dependent-chain microbenchmark tools/micro/latency.cu
# -> profiles/latency_r02.json; the guide's B300 numbers are the fallback.
# "global_coalesced" is an L2 hit (the halo rows a neighbouring tile fetched),
# "global_uncoalesced" one warp load touching 32 sectors.
_FALLBACK_LATENCY = {"register": 8, "shared": 29, "l1": 32, "global_coalesced": 250,
                     "global_uncoalesced": 1000, "dram": 580}


def _measured_latency() -> tuple[dict, str]:
    p = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                     "latency_r02.json")
    try:
        with open(p) as fh:
            m = json.load(fh)
        return {"register": m["register"], "shared": m["shared"], "l1": m["l1"],
                "global_coalesced": m["l2"], "global_uncoalesced": m["global_uncoalesced"],
                "dram": m["dram"]}, "measured (profiles/latency_r02.json)"
    except (OSError, KeyError, ValueError):
        return dict(_FALLBACK_LATENCY), "fallback (B300 guide)"


LATENCY, LATENCY_SOURCE = _measured_latency()


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
GRID_C = 162 ** 3                 # BT class C points (the tuned workload)
SMSPS = 148 * 4                   # SM sub-partitions (schedulers)
CLOCK_GHZ = 1.75                  # SM clock under the 1 kW power cap (bench clocks)
SMEM_CARVEOUTS_KB = (0, 8, 16, 32, 64, 100, 132, 164, 196, 228)
# Calibration of the two empirical terms (one measurement each):
ETA = 0.78       # issue efficiency vs the STATIC step body (fit: default variant 134 us)
GAMMA = 0.25     # share of non-FP64 instructions left exposed (3-4 warps per scheduler)
T_FACE_92 = 108.0  # us, boundary-face CTAs with a 92 KB L1 (profiles/timeline_ws_r02.txt)
FACE_EXP = 0.65  # L1 sensitivity of the face CTAs (fit: 142 us at 60 KB, 205 us at 28 KB)


@dataclasses.dataclass(frozen=True)
class Variant:
    """One point of the kernel family.  ws: where the step-0 fields rho_i /
    square live -- 0 recomputed per use in registers (round-1 kernel), 1
    evaluated once per point by a producer warpgroup into a shared-memory
    ring (rhs_ws.cuh); ring / fring: TMA ring depths (u, forcing); xoreg:
    edge-tile case bits register-resident; ty: tile rows; strict: the
    bit-identical contract (no FMA contraction)."""
    ws: int = 1
    ring: int = 4
    fring: int = 2
    xoreg: int = 1
    ty: int = 12
    strict: int = 0
    rcp: int = 2

    @property
    def threads(self) -> int:
        return 32 * (self.ty + (4 if self.ws else 0))

    @property
    def reg_limit(self) -> int:
        if self.ws:  # consumers after setmaxnreg (producers keep 32)
            return min(255, ((2048 - 4 * 32) // self.ty) // 8 * 8)
        return min(255, (65536 // self.threads) // 8 * 8)

    @property
    def smem_bytes(self) -> int:
        tx, hx = 32, 3
        ux, uy = tx + 2 * hx, self.ty + 4
        u_slot = ((ux * uy * 5 * 8 + 127) // 128) * 128
        f_slot = (((tx + 2) * self.ty * 5 * 8 + 127) // 128) * 128
        if self.ws:
            aux = ((self.ring * (tx + 2) * (self.ty + 2) * 16 + 127) // 128) * 128
            return self.ring * u_slot + aux + self.fring * f_slot + (3 * self.ring + 2 * self.fring) * 8
        return self.ring * (u_slot + f_slot) + (16 + 3 * tx + tx // 2) * 8

    @property
    def l1_kb(self) -> int:
        need = (self.smem_bytes + 1024 + 1023) // 1024  # + 1 KB reserved per CTA
        carve = next(c for c in SMEM_CARVEOUTS_KB if c >= need) if need <= 228 else 228
        return 256 - carve

    def defines(self) -> list[str]:
        d = [f"-DSAFARA_TY={self.ty}", f"-DSAFARA_RCP={self.rcp}"]
        if self.ws:
            d += [f"-DSAFARA_WS_US={self.ring}", f"-DSAFARA_WS_FS={self.fring}",
                  f"-DSAFARA_WS_XOREG={self.xoreg}"]
        else:
            d += [f"-DSAFARA_STAGES={self.ring}"]
        return d

    def env(self) -> dict:
        return {"SAFARA_WS": str(self.ws)}

    def kernel(self) -> str:
        v = "strict" if self.strict else "fast"
        name = f"rhs_kernel_{v}_ws_ud" if self.ws else f"rhs_kernel_{v}_ud"
        return f"_ZN6safara{len(name)}{name}E14CUtensorMap_stS0_NS_6ParamsE"

    def tag(self) -> str:
        t = (f"ws_u{self.ring}f{self.fring}x{self.xoreg}" if self.ws else f"r1_s{self.ring}")
        t += f"_ty{self.ty}" if self.ty != 12 else ""
        return t + ("_strict" if self.strict else "")


def default_family() -> list[Variant]:
    """Aux placement x ring depths x register residency x contract: ten
    variants (SURVEY §8(f) f3's knobs; tile width is fixed by the warp)."""
    return [Variant(ws=1, ring=4, fring=2, xoreg=1), Variant(ws=1, ring=4, fring=2, xoreg=0),
            Variant(ws=1, ring=4, fring=4), Variant(ws=1, ring=5, fring=2),
            Variant(ws=1, ring=3, fring=2), Variant(ws=0, ring=4), Variant(ws=0, ring=5),
            Variant(ws=0, ring=4, ty=8), Variant(ws=1, ring=4, fring=2, strict=1),
            Variant(ws=0, ring=4, strict=1)]


_FP64 = ("DFMA", "DMUL", "DADD")


def sass_loop_stats(obj: str, fn: str) -> dict | None:
    """Per-point instruction mix of the kernel's k march, read from the SASS
    of a compiled variant (the compile feedback, as SAFARA reads ptxas):
    the largest backward-branch loop that contains FP64 work, 3 steps per
    body (the register-renaming unroll)."""
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", "-fun", fn, obj],
                          capture_output=True, text=True).stdout
    ins = []
    for line in sass.splitlines():
        m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
        if m:
            ins.append((int(m.group(1), 16), m.group(2).strip()))
    if not ins:
        return None
    # out-of-line stubs (mbarrier retry blocks) sit after the last EXIT and
    # branch back into the body: they are not loops
    last_exit = max((i for i, (_, t) in enumerate(ins) if "EXIT" in t), default=len(ins) - 1)
    ins = ins[:last_exit + 1]
    # the k march: the innermost loop holding at least three steps' FP64 work
    best = None
    for a, t in ins:
        m = re.search(r"BRA(?:\.\w+)? 0x([0-9a-f]+)", t)
        if m and int(m.group(1), 16) < a:
            lo = int(m.group(1), 16)
            body = [x for y, x in ins if lo <= y <= a]
            nfp = sum(1 for x in body if re.sub(r"^@!?U?P\w+\s+", "", x).split()[0].split(".")[0]
                      in _FP64)
            if nfp >= 600 and (best is None or len(body) < len(best)):
                best = body
    if best is None:
        return None
    ops = [re.sub(r"^@!?U?P\w+\s+", "", x).split()[0].split(".")[0] for x in best]
    steps = 3
    return {"fp64": sum(o in _FP64 for o in ops) / steps,
            "lds": sum(o == "LDS" for o in ops) / steps,
            "local": sum(o in ("STL", "LDL") for o in ops) / steps,
            "other": sum(o not in _FP64 for o in ops) / steps,
            "body_instructions": len(best)}


def compile_variant(v: Variant, workdir: str) -> dict:
    """nvcc the variant's translation unit with its defines; ptxas feedback
    (registers, spill bytes) and the SASS mix of its k march."""
    from . import build as b
    unit = "rhs_strict.cu" if v.strict else "rhs_fast.cu"
    obj = os.path.join(workdir, v.tag() + ".o")
    cmd = [b.NVCC, *b.COMMON, "--fmad=false" if v.strict else "--fmad=true", "-Xptxas", "-v",
           *v.defines(), "-c", os.path.join(b.CSRC, unit), "-o", obj]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        return {"variant": v, "error": res.stderr[-400:]}
    info = ptxas_info(res.stdout + res.stderr)
    return {"variant": v, "kernels": info, "prod": info.get(v.kernel()),
            "sass": sass_loop_stats(obj, v.kernel())}


def model_cost(v: Variant, regs: int, spill_bytes: int = 0, sass: dict | None = None,
               latency: dict = LATENCY) -> float:
    """Predicted BT class C pass time (us) of a variant.

    Compute: the k march issues F FP64 and O other warp-instructions per
    point (SASS of the variant); the FP64 pipe takes 2 cycles per warp
    instruction, the scheduler 1 per cycle, so one point costs
    (max(2F, F+O) + GAMMA*O)/32 scheduler cycles (static counts of the step
    body: both sides of the edge/mid branches) at the calibrated issue
    efficiency ETA;
    spills add their local-memory round trips at the measured L1 latency
    (ptxas spill bytes / 8 accesses if the SASS has none in the loop).
    Registers: a variant over its budget cannot launch (infinite cost).
    Grid: the lockstep schedule's busy SMs (ncol tiles x k-parts) relative to
    the calibrated 140; TMA lookahead below 2 steps exposes one DRAM latency
    (measured table) per step of the march.
    Boundary faces: the face CTAs' strided column gathers are L1-bound:
    T_FACE_92 * (92 KB / L1 KB)^FACE_EXP (calibrated; the carveout a
    variant's shared memory leaves decides the L1).  The pass takes the
    longer of the two."""
    if regs > v.reg_limit:
        return float("inf")
    if sass is None:
        return float("inf")
    F, O = sass["fp64"], sass["other"]
    local = sass["local"] if sass["local"] else spill_bytes / 8 / 3
    c_issue = (max(2 * F, F + O) + GAMMA * O) / 32.0
    c_spill = local * latency["l1"] / 32.0
    t_compute = (GRID_C / SMSPS) * (c_issue / ETA + c_spill) / (CLOCK_GHZ * 1e3)
    # lockstep grid: ncol column tiles x floor(148 / ncol) k-parts; fewer
    # busy SMs than the calibrated 12-row shape (140 CTAs) stretch the pass
    ncol = -(-160 // 32) * -(-160 // v.ty)
    ctas = ncol * max(1, 148 // ncol) if ncol <= 148 else 148
    t_compute *= 140.0 / min(ctas, 148)
    # TMA lookahead: a plane is requested ring-2 steps before its own column
    # is read; with less than 2 steps one DRAM round trip per step is exposed
    look = v.ring - 2
    steps = 160 / max(1, 148 // ncol)
    t_compute += max(0, 2 - look) * steps * latency["dram"] / (CLOCK_GHZ * 1e3)
    t_face = T_FACE_92 * (92.0 / max(v.l1_kb, 1)) ** FACE_EXP
    return max(t_compute, t_face)


def tune_variants(family=None, jobs: int = 4) -> list[dict]:
    """Compile the family, apply SAFARA's feasibility rule (no spills, within
    the register budget of the CTA shape) and rank by the
    model."""
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
        spill = p["spill_st"] + p["spill_ld"]
        ok = spill == 0 and p["regs"] <= v.reg_limit
        rows.append({"variant": v.tag(), "defines": v.defines(), "env": v.env(),
                     "strict": v.strict, "regs": p["regs"], "reg_limit": v.reg_limit,
                     "spill_bytes": spill, "smem_kb": round(v.smem_bytes / 1024, 1),
                     "l1_kb": v.l1_kb, "sass": r.get("sass"), "feasible": ok,
                     "model_us": round(model_cost(v, p["regs"], spill, r.get("sass")), 1)})
    rows.sort(key=lambda r: (not r.get("feasible", False), r.get("model_us", 1e9)))
    return rows


def register_feedback(jobs: int = 2) -> dict:
    """SAFARA's loop (feedback_loop) run against real compiles of the
    warp-specialised consumer: the candidate is the edge tiles' xi case
    bits (reuse: every step of an edge tile; replacing them by a register
    saves their recomputation, ~10 integer instructions at register
    latency each).  compile_regs builds the variant and reports the
    registers the consumer demands (ptxas count + spilled words)."""
    cand = [Candidate("xi_case_bits", uses=10, space="register", regs=1)]
    lat = dict(LATENCY)
    lat["register"] = max(lat["register"], 1)

    def compile_regs(names):
        v = Variant(ws=1, xoreg=1 if "xi_case_bits" in names else 0)
        with tempfile.TemporaryDirectory() as wd:
            r = compile_variant(v, wd)
        p = r["prod"]
        return p["regs"] + (p["spill_st"] + p["spill_ld"]) // 4

    limit = Variant(ws=1).reg_limit + 4  # registers + a word of slack
    chosen, hist = feedback_loop(cand, compile_regs, limit, lat)
    return {"chosen": [c.name for c in chosen], "history": hist, "limit": limit}


def time_variant(v: Variant, steps: int = 200, libdir: str | None = None) -> float | None:
    """Build the full library for a variant and time it with bench.py (GPU)."""
    from . import build as b
    libdir = libdir or os.path.join(b.ROOT, "ablibs")
    out = os.path.join(libdir, f"tune_{v.tag().replace('_strict', '')}.so")
    if not os.path.exists(out):
        b.build(force=True, extra=v.defines(), out=out,
                objdir=os.path.join(libdir, "obj_tune_" + v.tag()))
    env = dict(os.environ, SAFARA_LIB=out, **v.env())
    cmd = [sys.executable, os.path.join(b.ROOT, "bench.py"), "--steps", str(steps),
           "--warmup", "10", "--no-cpu-baseline", "--no-other-configs", "--soak-s", "0.5",
           "--e2e-steps", "0"] + (["--strict"] if v.strict else [])
    res = subprocess.run(cmd, capture_output=True, text=True, env=env)
    try:
        return json.loads(res.stdout.strip().splitlines()[-1])["roofline"]["kernel_ms"] * 1e3
    except Exception:
        return None


def main(argv=None):
    ap = argparse.ArgumentParser(description=__doc__.split("\n\n")[0])
    ap.add_argument("--build", action="store_true",
                    help="also build each variant's library into ablibs/ (for --time on a GPU box)")
    ap.add_argument("--time", type=int, default=0, help="time every variant N times (GPU)")
    ap.add_argument("--jobs", type=int, default=4)
    a = ap.parse_args(argv)
    print(json.dumps({"latency": LATENCY, "source": LATENCY_SOURCE}))
    rows = tune_variants(jobs=a.jobs)
    for r in rows:
        print(json.dumps(r))
    print(json.dumps({"register_feedback": register_feedback()}))
    fam = {v.tag(): v for v in default_family()}
    if a.build:
        from . import build as b
        libdir = os.path.join(b.ROOT, "ablibs")
        os.makedirs(libdir, exist_ok=True)

        def one(v):
            out = os.path.join(libdir, f"tune_{v.tag().replace('_strict', '')}.so")
            if not os.path.exists(out):
                b.build(force=True, extra=v.defines(), out=out,
                        objdir=os.path.join(libdir, "obj_tune_" + v.tag()))
            return out
        with cf.ThreadPoolExecutor(a.jobs) as ex:
            list(ex.map(one, [v for v in fam.values() if not v.strict]))
    if a.time:
        meas = {}
        for rep in range(a.time):
            for r in rows:
                if "error" in r:
                    continue
                us = time_variant(fam[r["variant"]])
                meas.setdefault(r["variant"], []).append(us)
                print(json.dumps({"variant": r["variant"], "rep": rep, "kernel_us": us}),
                      flush=True)
        best = {k: min(x for x in t if x) for k, t in meas.items() if any(t)}
        fastest = min(best, key=best.get)
        pick = next(r["variant"] for r in rows if r.get("feasible"))
        print(json.dumps({"model_pick": pick, "fastest_measured": fastest,
                          "match": pick == fastest, "measured_min_us": best}))


if __name__ == "__main__":
    main()
