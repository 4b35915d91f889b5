"""The generated inline-PTX includes are in step with their generators (scripts/gen_*.py):
regenerating into a temporary file reproduces the committed csrc/*.inc byte for byte, so the
kernels that are built are the ones the generators (and DESIGN.md §3.4) describe."""
import importlib.util
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_middleware_hafeezsg021_b200", "csrc")


@pytest.mark.parametrize("gen, inc", [("gen_fast_walk.py", "fast_walk_ptx.inc"),
                                      ("gen_uni_push.py", "uni_push_ptx.inc")])
def test_generated_ptx_in_sync(tmp_path, gen, inc, capsys):
    spec = importlib.util.spec_from_file_location(gen[:-3], os.path.join(ROOT, "scripts", gen))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    out = tmp_path / inc
    mod.OUT = str(out)
    mod.main()
    committed = open(os.path.join(CSRC, inc)).read()
    assert out.read_text() == committed, f"{inc} is stale: run python scripts/{gen}"
