"""NEXT-2 spill I/O path on the CPU (no GPU): the O_DIRECT io_uring transfers the spill tier uses,
exercised through sh_spill_probe on a fresh file (write, fdatasync, read back)."""
import pytest

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")


def test_spill_probe_roundtrip(tmp_path):
    r = sh.spill_probe(str(tmp_path), 64 << 20)
    assert r["read_gbs"] > 0 and r["write_gbs"] > 0
    assert list(tmp_path.iterdir()) == []  # unlinked at creation


def test_spill_probe_bad_dir(tmp_path):
    with pytest.raises(sh.ShError):
        sh.spill_probe(str(tmp_path / "missing"), 1 << 20)
