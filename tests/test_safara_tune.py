"""SAFARA's selection and feedback loop (§III-B)
and the variant tuner's ptxas feedback, on the CPU."""
import pytest

from paper_conf_icpp_tiankexc16_b200 import safara_tune as st

# PAPER.md Fig. 5 (L650-668): in the sequential i loop, the a group
# (a[i-1][j], a[i][j] read+write, a[i+1][j]) is coalesced across the j
# threads; the b group (b[j][i-1], b[j][i+1], plus b[j][0], b[j][1] above)
# is uncoalesced.  Each needs 3 temporaries (L674-676); a is used once more.
A = st.Candidate("a", uses=4, space="global_coalesced", regs=3)
B = st.Candidate("b", uses=3, space="global_uncoalesced", regs=3)


def test_running_example_26_of_30_registers_selects_b():
    """L872-893: 26 registers used, limit 30 -> 4 available -> the scalar
    replacement is applied to array b with 3 registers (Fig. 6)."""
    chosen, free = st.select([A, B], used=26, limit=30)
    assert [c.name for c in chosen] == ["b"]
    assert free == 1


def test_carr_kennedy_count_only_would_pick_a():
    """With latency ignored (the CPU cost model, L670-689), a wins on count."""
    flat = {k: 1 for k in st.LATENCY}
    chosen, _ = st.select([A, B], used=26, limit=30, latency=flat)
    assert [c.name for c in chosen] == ["a"]


def test_enough_registers_takes_both_and_none_when_full():
    chosen, free = st.select([A, B], used=20, limit=30)
    assert {c.name for c in chosen} == {"a", "b"} and free == 4
    assert st.select([A, B], used=29, limit=30)[0] == []


def test_feedback_loop_iterates_until_saturated():
    """Compile -> registers -> select, one group per round (L727-736)."""
    calls = []

    def compile_regs(names):
        calls.append(names)
        return 26 + 3 * len(names)

    chosen, hist = st.feedback_loop([A, B], compile_regs, limit=30)
    assert [c.name for c in chosen] == ["b"]
    assert [h[2] for h in hist] == [26, 29]
    assert calls == [(), ("b",)]


PTXAS_LOG = """\
ptxas info    : Compiling entry function '_ZN6safara18rhs_kernel_fast_udE14CUtensorMap_stS0_NS_6ParamsE' for 'sm_100a'
ptxas info    : Function properties for _ZN6safara18rhs_kernel_fast_udE14CUtensorMap_stS0_NS_6ParamsE
    0 bytes stack frame, 0 bytes spill stores, 0 bytes spill loads
ptxas info    : Used 168 registers, used 1 barriers, 128 bytes smem
ptxas info    : Compiling entry function 'k2' for 'sm_100a'
    8 bytes stack frame, 4 bytes spill stores, 12 bytes spill loads
ptxas info    : Used 255 registers, used 1 barriers
"""


def test_ptxas_parser():
    info = st.ptxas_info(PTXAS_LOG)
    prod = info["_ZN6safara18rhs_kernel_fast_udE14CUtensorMap_stS0_NS_6ParamsE"]
    assert prod == {"regs": 168, "spill_st": 0, "spill_ld": 0, "stack": 0}
    assert info["k2"] == {"regs": 255, "spill_st": 4, "spill_ld": 12, "stack": 8}


def test_variant_register_budget():
    assert st.Variant(ws=0, ty=12).reg_limit == 168
    assert st.Variant(ws=0, ty=8).reg_limit == 255
    assert st.Variant(ws=0, ty=10).reg_limit == 200
    # warp-specialised: 12 consumer warps share what 4 producer warps at 32
    # registers leave of the 64K file
    assert st.Variant(ws=1).reg_limit == 160


def test_variant_shared_memory_matches_the_kernel_constants():
    """safara_internal.h: SMEM_BYTES = 4 slots x (u 24320 + forcing 16384) +
    1 KB of barriers/table; WS_SMEM_BYTES = u 4 x 24320 + aux 4 x 7616 +
    forcing 2 x 16384 + 16 barriers -> both leave the 92 KB L1 of a 164 KB
    carveout; 5-slot rings cross into the 196 / 228 KB carveouts."""
    assert st.Variant(ws=0, ring=4).smem_bytes == 163840
    assert st.Variant(ws=1, ring=4, fring=2).smem_bytes == 160640
    assert st.Variant(ws=0, ring=4).l1_kb == 92 and st.Variant(ws=1).l1_kb == 92
    assert st.Variant(ws=0, ring=5).l1_kb == 28
    assert st.Variant(ws=1, ring=4, fring=4).l1_kb == 60


def test_latency_table_is_measured():
    """The L of L x C comes from the B200 microbenchmark."""
    assert st.LATENCY_SOURCE.startswith("measured")
    L = st.LATENCY
    assert L["register"] < L["shared"] < L["l1"] < L["global_coalesced"] < L["dram"]


def test_tune_compiles_and_ranks_two_variants():
    """Real nvcc + ptxas + SASS feedback for two variants (cross-compiles, no
    GPU): both spill-free and within budget; the warp-specialised kernel's
    k march has fewer FP64 and other instructions per step and ranks first
    (measured on B200: 134.9 vs 142.2 us, profiles/safara_tune_r02.txt)."""
    rows = st.tune_variants([st.Variant(ws=1), st.Variant(ws=0)], jobs=2)
    assert len(rows) == 2
    for r in rows:
        assert "error" not in r, r
        assert r["feasible"] and r["spill_bytes"] == 0
        assert r["sass"]["fp64"] > 200 and r["sass"]["local"] == 0
    assert rows[0]["variant"] == "ws_u4f2x1"
    ws, r1 = rows
    assert ws["sass"]["fp64"] < r1["sass"]["fp64"]
    assert ws["sass"]["body_instructions"] < r1["sass"]["body_instructions"]
    assert ws["model_us"] < r1["model_us"]


def test_model_penalises_small_l1_spills_and_short_rings():
    sass = {"fp64": 375.0, "other": 268.0, "local": 0.0}
    base = st.model_cost(st.Variant(ws=1), 128, 0, sass)
    assert st.model_cost(st.Variant(ws=1, fring=4), 128, 0, sass) > base      # L1 60 KB
    assert st.model_cost(st.Variant(ws=1, ring=3), 128, 0, sass) > base       # 1 step lookahead
    assert st.model_cost(st.Variant(ws=1), 128, 0, dict(sass, local=3.0)) > base
    assert st.model_cost(st.Variant(ws=1), 999, 0, sass) == float("inf")     # over budget
