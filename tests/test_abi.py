"""The C-ABI library loads and exports every symbol include/dts.h declares;
host-side validation and the no-GPU failure mode (CPU only, no compute)."""
import ctypes as C
import os
import re

import numpy as np
import pytest

import gen
import paper_conf_ipps_gonthiermt22_b200 as dts
from paper_conf_ipps_gonthiermt22_b200 import dts as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "dts.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(dts_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    lib = dts.load_library()
    names = _declared()
    assert "dts_instance_create" in names and "dts_run" in names and "dts_result" in names
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(dts.EXPORTED) == names


def test_struct_layouts():
    assert dts.EVENT_DTYPE.itemsize == 32
    assert C.sizeof(B.dts_run_opts) == 48
    assert dts.dts_version() >> 16 == 1


def test_struct_layouts_match_the_header(tmp_path):
    """The binding's ctypes mirrors against the C compiler's view of include/dts.h:
    size of every struct and the offset of every field (gcc, no GPU)."""
    import subprocess
    structs = {"dts_run_opts": B.dts_run_opts, "dts_result_view": B.dts_result_view}
    lines = ["#include <stdio.h>", "#include <stddef.h>", '#include "dts.h"', "int main(void) {"]
    for name, cls in structs.items():
        lines.append(f'printf("{name} %zu\\n", sizeof({name}));')
        for f, _ in cls._fields_:
            lines.append(f'printf("{name}.{f} %zu\\n", offsetof({name}, {f}));')
    lines.append('printf("dts_event %zu\\n", sizeof(dts_event)); return 0; }')
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = dict(l.split() for l in subprocess.check_output([str(exe)], text=True).splitlines())
    for name, cls in structs.items():
        assert int(got[name]) == C.sizeof(cls), name
        for f, _ in cls._fields_:
            assert int(got[f"{name}.{f}"]) == getattr(cls, f).offset, f"{name}.{f}"
    assert int(got["dts_event"]) == dts.EVENT_DTYPE.itemsize


def test_opts_defaults():
    o = dts.dts_run_opts_default()
    assert o.flags == dts.DTS_F_FALLBACK2 and o.lookahead_W == 0
    assert o.bus_bytes_per_s == 12_000_000_000 and o.max_served == -1


@pytest.mark.parametrize("bad,status", [
    (dict(K=0), B.DTS_E_INVAL),
    (dict(K=65), B.DTS_E_UNSUPPORTED),
    (dict(task_data=np.array([0, 9, 1, 2], np.int32)), B.DTS_E_INVAL),
    (dict(task_ptr=np.array([0, 3, 2], np.int64), task_data=np.array([0, 1, 1], np.int32)), B.DTS_E_INVAL),
    # an inner entry past E = task_ptr[m]: rejected before any row is read
    (dict(task_ptr=np.array([0, 5, 2], np.int64), task_data=np.array([0, 1], np.int32)), B.DTS_E_INVAL),
    (dict(data_size=np.array([1, 0, 1], np.uint64)), B.DTS_E_INVAL),
])
def test_validation(bad, status):
    args = dict(task_ptr=np.array([0, 2, 4], np.int64), task_data=np.array([0, 1, 1, 2], np.int32),
                data_size=np.ones(3, np.uint64), task_ns=None, default_task_ns=1,
                mem_capacity_bytes=2, K=1)
    args.update(bad)
    with pytest.raises(dts.DtsError) as e:
        dts.dts_instance_create(**args)
    assert e.value.status == status


def test_too_many_inputs_unsupported():
    tp = np.array([0, 128], np.int64)
    td = np.arange(128, dtype=np.int32)
    with pytest.raises(dts.DtsError) as e:
        dts.dts_instance_create(tp, td, np.ones(128, np.uint64), None, 1, 200, 1)
    assert e.value.status == B.DTS_E_UNSUPPORTED


def test_capacity_checked_before_device():
    i = gen.fig1()
    h = dts.dts_instance_create(i.task_ptr, i.task_data, i.data_size, None, 1, 1, 2)  # M=1 < 2 inputs
    with pytest.raises(dts.DtsError) as e:
        dts.dts_run(h)
    assert e.value.status == B.DTS_E_CAPACITY


def test_result_before_run_is_state_error():
    i = gen.fig1()
    h = dts.dts_instance_create(i.task_ptr, i.task_data, i.data_size, None, 1, 2, 2)
    with pytest.raises(dts.DtsError) as e:
        dts.dts_result(h)
    assert e.value.status == B.DTS_E_STATE


def test_unsupported_options():
    i = gen.fig1()
    h = dts.dts_instance_create(i.task_ptr, i.task_data, i.data_size, None, 1, 4, 2)
    with pytest.raises(dts.DtsError) as e:
        dts.dts_run(h, opts=dts.dts_run_opts_default(lookahead_W=9))  # taskBuffer > 9 tasks
    assert e.value.status == B.DTS_E_UNSUPPORTED


def test_no_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    i = gen.fig1()
    with pytest.raises(dts.DtsError) as e:
        dts.schedule(i)
    assert e.value.status == B.DTS_E_CUDA


def test_fetch_results_before_run_is_state_error():
    i = gen.fig1()
    hs = [dts.dts_instance_create(i.task_ptr, i.task_data, i.data_size, None, 1, 2, 2) for _ in range(2)]
    with pytest.raises(dts.DtsError) as e:
        dts.dts_fetch_results(hs)
    assert e.value.status == B.DTS_E_STATE
    dts.dts_fetch_results([])  # nothing to do
