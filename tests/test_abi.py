"""The C-ABI library loads on a CPU-only box and exports every symbol include/deepplan.h
declares (no GPU compute is called here)."""
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "deepplan.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+char\s*\*|dp_status|int32_t|int64_t)\s+(dp_[a-z0-9_]+)\s*\(",
                                 src, flags=re.M)))


def test_header_declares_the_boundary():
    names = _declared()
    for must in ("dp_plan_generate", "dp_plan_simulate", "dp_profile", "dp_infer_cold", "dp_infer_warm",
                 "dp_model_create", "dp_serve_run", "dp_embed", "dp_linear", "dp_peer_init"):
        assert must in names


def test_library_exports_every_declared_symbol():
    import paper_conf_eurosys_jeongba23_b200 as dp
    for name in _declared():
        assert hasattr(dp.lib, name), name
    assert dp.lib.dp_abi_version() == 2


def test_error_path_sets_last_error():
    import paper_conf_eurosys_jeongba23_b200 as dp
    import pytest
    with pytest.raises(dp.DeepPlanError) as e:
        dp.plan_partition([1, 2, 3], 0)  # k must be >= 1
    assert "k out of range" in str(e.value)


def test_config_params_match_synth_names():
    import synth
    from paper_conf_eurosys_jeongba23_b200._lib import config_params
    for name in ("tiny_bert", "tiny_roberta", "tiny_gpt2", "bert_base", "gpt2_medium"):
        m = synth.SHAPES[name]
        ps = config_params(m)
        hf = synth.hf_param_shapes(m)
        assert [p["name"] for p in ps] == list(hf.keys())
        assert [p["shape"] for p in ps] == list(hf.values())
