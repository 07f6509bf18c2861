"""tools/timeline.py (bench.py --timeline) on a hand-made CUPTI-style trace: busy time per
activity and the overlap of the miss stream with sampling (interval arithmetic)."""
import json

from tools.timeline import summarise


def test_overlap_accounting(tmp_path):
    ev = [  # ts, dur in us
        {"cat": "kernel", "name": "void gd::k_sample_hop<8, 128>(gd::SampleHopArgs)", "ts": 0, "dur": 100, "args": {"stream": 7}},
        {"cat": "kernel", "name": "void gd::k_relabel_hop(gd::RelabelArgs)", "ts": 100, "dur": 50, "args": {"stream": 7}},
        {"cat": "kernel", "name": "void gd::k_miss_copy<4, 0>(...)", "ts": 50, "dur": 200, "args": {"stream": 9}},
        {"cat": "gpu_memcpy", "name": "Memcpy HtoD (Pinned -> Device)", "ts": 120, "dur": 100, "args": {"stream": 11}},
        {"cat": "kernel", "name": "void gd::k_lookup(gd::LookupArgs)", "ts": 160, "dur": 40, "args": {"stream": 7}},
        {"cat": "kernel", "name": "at::native::fill_kernel", "ts": 0, "dur": 400, "args": {"stream": 7}},   # not ours
    ]
    p = tmp_path / "t.json"
    p.write_text(json.dumps({"traceEvents": ev}))
    out = tmp_path / "t.md"
    r = summarise(str(p), str(out), 2, "test")
    assert r["window_ms"] == 0.25                      # 0 .. 250 us (torch's fill ignored)
    # miss union = [50, 250] = 200 us; sampling = [0, 150]; overlap = [50, 150] = 100 us
    assert r["miss_busy_ms"] == 0.2 and r["miss_overlapped_with_sampling_ms"] == 0.1
    assert r["miss_overlap_share"] == 0.5
    text = out.read_text()
    assert "miss copy-engine H2D" in text and "```" in text
