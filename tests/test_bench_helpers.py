"""bench.py's host-side helpers (CPU): the roofline traffic capture it picks and the oracle sample's skip
list.  The bench itself needs a GPU; these pieces decide what its JSON line reports."""
import json

import bench


def _write(d, name, **kw):
    (d / name).write_text(json.dumps(kw))


def test_load_traffic_prefers_a_capture_of_the_running_sources(tmp_path, monkeypatch):
    prof = tmp_path / "profiles"
    prof.mkdir()
    monkeypatch.setattr(bench, "ROOT", str(tmp_path))
    here = bench.source_hash()   # no engine sources under tmp_path: the hash of nothing, still a fixed value
    _write(prof, "r02x_batch_traffic.json", workload="C4", src_sha256="old", captured_unix=200,
           dram_bytes_per_query=2.0, git_sha="x")
    _write(prof, "r02_batch_traffic.json", workload="C4", src_sha256=here, captured_unix=100,
           dram_bytes_per_query=1.0, git_sha="y")
    _write(prof, "r02z_batch_traffic.json", workload="C3", src_sha256=here, captured_unix=300,
           dram_bytes_per_query=3.0, git_sha="z")
    b, info = bench.load_traffic("C4")
    assert b == 1.0 and info["traffic_source"] == "r02_batch_traffic.json" and info["traffic_matches_source"]
    # without a matching capture: the newest one, and it says so
    (prof / "r02_batch_traffic.json").unlink()
    _write(prof, "r01_batch_traffic.json", workload="C4", src_sha256="older", dram_bytes_per_query=5.0)
    b, info = bench.load_traffic("C4")
    assert b == 2.0 and info["traffic_source"] == "r02x_batch_traffic.json" and not info["traffic_matches_source"]
    assert bench.load_traffic("C5") == (None, {"traffic_source": None})


def test_oracle_skip_list_is_c4_level5_queries():
    skip = bench.ORACLE_SKIP["C4"]
    assert len(skip) == len(set(skip)) == 7 and all(0 <= i < 4096 for i in skip)
    assert bench.ORACLE_SKIP.get("C3", ()) == ()
