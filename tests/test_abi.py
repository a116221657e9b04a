"""The C-ABI library loads and exports every symbol include/psml.h declares (not gpu)."""
import re

import pytest

from paper_conf_icpp_chenzzzz020_b200 import build, psml


@pytest.fixture(scope="module")
def header_symbols():
    text = open(psml.HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(psml_[a-z0-9_]+)\s*\(", text)))


def test_library_builds_and_loads():
    path = build.build()
    assert path.endswith("libpsml.so")
    assert psml.abi_version() == 1


def test_every_declared_symbol_is_exported_and_bound(header_symbols):
    L = psml.lib()
    for name in header_symbols:
        assert hasattr(L, name), name
    assert sorted(psml.EXPORTS) == header_symbols


def test_no_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is visible")
    with pytest.raises(psml.PsmlError) as e:
        psml.Ctx()
    assert e.value.status == 4  # PSML_ERR_UNSUPPORTED, never a CPU fallback
    assert psml.msb_material_words(psml.Ring(64, 13), 10) == 11 * 10   # reduced prefix (R27)
    assert psml.msb_material_words(psml.Ring(32, 13), 10) == 11 * 10


def test_binding_rejects_wrong_buffers_before_the_abi():
    """the binding checks device, contiguity, dtype and element count before a
    pointer reaches the C ABI (which takes sizes from the model description)."""
    import torch
    from paper_conf_icpp_chenzzzz020_b200 import psml
    cpu = torch.zeros(4, dtype=torch.uint64)
    with pytest.raises(psml.PsmlError):
        psml._pair((cpu, cpu))
    with pytest.raises(psml.PsmlError):
        psml._check(torch.zeros(10, dtype=torch.uint64), 12, (torch.uint64,), "X")
    with pytest.raises(psml.PsmlError):
        psml._check(torch.zeros(12, dtype=torch.float64), 12, (torch.uint64,), "X")
    psml._check(torch.zeros(12, dtype=torch.uint64), 12, (torch.uint64,), "X")
