"""The C-ABI library loads and exports every symbol include/vista.h declares; host-only
entry points work without a GPU; compute entry points fail loudly (no CPU fallback)."""
import ctypes
import os
import re

import pytest

from conftest import ROOT, has_gpu

HDR = os.path.join(ROOT, "include", "vista.h")


def declared_functions():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(vista_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    f = declared_functions()
    for name in ["vista_plan", "vista_transfer", "vista_train", "vista_features", "vista_destroy"]:
        assert name in f


def test_library_exports_every_declared_symbol():
    from paper_conf_sigmod_nakandalak20_b200 import vista as V
    L = V.lib()
    missing = [n for n in declared_functions() if not hasattr(L, n)]
    assert not missing, missing


def test_shard_range_partitions_rows():
    from paper_conf_sigmod_nakandalak20_b200 import vista_shard_range
    for n in [0, 1, 7, 20000, 200001]:
        for world in [1, 2, 3, 8]:
            spans = [vista_shard_range(n, r, world) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == n
            for (a, b), (c, d) in zip(spans, spans[1:]):
                assert b == c and a <= b
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= 1


def test_status_strings():
    from paper_conf_sigmod_nakandalak20_b200 import vista as V
    assert V.lib().vista_status_str(2) == b"no feasible plan within the HBM budget"


@pytest.mark.skipif(has_gpu(), reason="checks the no-GPU error path")
def test_no_cpu_fallback_without_gpu():
    from paper_conf_sigmod_nakandalak20_b200 import Vista, VistaError
    with pytest.raises(VistaError) as e:
        Vista(0, layers=[0], n_str_rows=4, d_s=8, n_images_local=4)
    assert e.value.status == 5


def test_invalid_arguments_rejected_before_gpu_work():
    from paper_conf_sigmod_nakandalak20_b200 import Vista, VistaError
    with pytest.raises(VistaError) as e:
        Vista(7, layers=[0], n_str_rows=4, d_s=8, n_images_local=4)
    assert e.value.status == 1
    with pytest.raises(VistaError) as e:
        Vista(0, layers=[2, 1], n_str_rows=4, d_s=8, n_images_local=4)
    assert e.value.status == 1
