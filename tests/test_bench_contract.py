"""Host-side checks of bench.py's contract (no GPU): defaults and the profile files
the roofline line reads."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _parse(argv):
    sys.path.insert(0, ROOT)
    import bench
    old = sys.argv
    try:
        sys.argv = ["bench.py"] + argv
        return bench.parse()
    finally:
        sys.argv = old


def test_defaults_follow_the_timing_rules():
    a = _parse([])
    assert a.gpus == 1 and a.warmup >= 3 and a.steps >= 1
    assert a.impl == "dycuckoo" and a.config == "c2"
    assert a.log2n == 27                       # BASELINE.json configs[1]


def test_roofline_traffic_pointer_names_an_existing_capture():
    pdir = os.path.join(ROOT, "profiles")
    latest = json.load(open(os.path.join(pdir, "traffic_latest.json")))
    tr = json.load(open(os.path.join(pdir, latest["file"])))
    # the dominant C2 kernel and the other probe kernels were captured
    for k in ("k_upsert", "k_find", "k_delete", "k_place"):
        assert tr[k] > 0
    assert os.path.exists(os.path.join(pdir, f"{latest['tag']}_summary.md"))
