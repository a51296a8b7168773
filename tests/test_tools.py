"""Host-side helpers of the measurement (no GPU): the L2-gather roof the bench line reports beside the HBM
roofline and the fwd/rev classification of the ncu summaries (profiles/ncu_traffic.json feeds
roofline.traffic)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))


def test_l2_gather_roof_counts_gathers_per_format():
    import bench
    slots = 1 << 28
    v2 = bench.l2_op_roof(2.75, slots, 1.58, slots, 2)
    v3 = bench.l2_op_roof(0.48 * 4, slots, 0.44 * 4, slots, 3)
    g = v2["gather_gps"]
    assert abs(v2["fwd_floor_ms"] - 2 * slots / g / 1e6) < 1e-3      # page entry + unit word
    assert abs(v3["fwd_floor_ms"] - slots / g / 1e6) < 1e-3          # the entry alone
    assert abs(v2["rev_floor_ms"] - slots / g / 1e6) < 1e-3          # the state word
    assert v2["fwd_frac"] == round(v2["fwd_floor_ms"] / 2.75, 4)
    assert "unit word" in v2["fwd_ops_per_slot"] and "unit word" not in v3["fwd_ops_per_slot"]


def test_ncu_kernel_classification():
    import ncu_summary as ns
    assert ns.kind_of("void cgcm::k_fwd_fast<(bool)1, (bool)0, (bool)0>(cgcm::SlotArgs)") == "fwd"
    assert ns.kind_of("void cgcm::k_rev_fast<(bool)1, (bool)1>(cgcm::SlotArgs)") == "rev"
    assert ns.kind_of("void cgcm::k_map_pd<1>(cgcm::SlotArgs)") == "fwd"
    assert ns.kind_of("void cgcm::k_unmap_sh<89, false>(cgcm::SlotArgs)") == "rev"
    assert ns.kind_of("void cgcm::k_slots<1, 89, 3, 1>(cgcm::SlotArgs)") == "rev"
    assert ns.kind_of("void cgcm::k_slots<0, 67, 3, 1>(cgcm::SlotArgs)") == "fwd"
