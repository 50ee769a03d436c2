"""The C-ABI library loads and exports every symbol include/ffs.h declares (CPU only:
no compute call is made without a GPU)."""
import ctypes
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared():
    src = open(os.path.join(ROOT, "include", "ffs.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ffs_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_survey_calls():
    names = declared()
    for n in ("ffs_create", "ffs_destroy", "ffs_last_error", "ffs_stage_tables", "ffs_plan_batch",
              "ffs_plan_keys", "ffs_plan_decode", "ffs_evict_scores"):
        assert n in names


def test_library_exports_every_declared_symbol():
    from paper_conf_hpdc_hui0s25_b200 import build
    lib = ctypes.CDLL(build.build())
    for n in declared():
        assert hasattr(lib, n), n


def test_binding_covers_every_declared_symbol():
    from paper_conf_hpdc_hui0s25_b200 import ffs
    assert sorted(ffs.EXPORTS) == declared()


def test_no_oracle_in_product_tree():
    pkg = os.path.join(ROOT, "paper_conf_hpdc_hui0s25_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "ffs_oracle" not in txt, f
