"""T0 (model level): the oracle's spec execution vs independent library models.

The spec + oracle composition of each config is pinned against the reference
architectures as implemented by torchvision (ResNet-50 v1.5, MobileNetV2) and
HF transformers (BertModel), run in float64 with the same weights (BatchNorm
set to an exact identity + bias), to ~1e-10 relative (SURVEY.md §8(c) "Library
pins").  A wrong residual wiring, stride placement, activation or head split
in either the spec or the oracle fails here.
"""
import numpy as np
import pytest
import torch

from oracle import models as om
from workloads import build_model


def _rel(a, b):
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-30))


def _set_conv(conv, bn, layer):
    conv.weight.data = torch.from_numpy(layer["w"].astype(np.float64))
    if bn is not None:
        bn.eps = 1e-300           # sqrt(1 + 1e-300) == 1 exactly in float64
        bn.running_mean.zero_()
        bn.running_var.fill_(1.0)
        bn.weight.data.fill_(1.0)
        bn.bias.data = torch.from_numpy(layer["b"].astype(np.float64))
    else:
        conv.bias.data = torch.from_numpy(layer["b"].astype(np.float64))


def test_tiny_cnn_vs_torch():
    spec, x = build_model("tiny_cnn")
    env = om.run_model(spec, x)
    convs = [l for l in spec["layers"] if l["op"] == "conv"]
    fc = [l for l in spec["layers"] if l["op"] == "linear"][0]
    t = torch.from_numpy(x.astype(np.float64))
    from oracle.ops import bf16_rne
    t = torch.from_numpy(bf16_rne(x))
    for c in convs:
        t = torch.relu(torch.nn.functional.conv2d(t, torch.from_numpy(c["w"].astype(np.float64)),
                                                  torch.from_numpy(c["b"].astype(np.float64)),
                                                  1, 1))
    t = torch.nn.functional.max_pool2d(t, 2, 2).flatten(1)
    t = torch.nn.functional.linear(t, torch.from_numpy(fc["w"].astype(np.float64)),
                                   torch.from_numpy(fc["b"].astype(np.float64)))
    t = torch.softmax(t, -1).numpy()
    assert _rel(env[spec["outputs"][0]], t) < 1e-12


@pytest.mark.slow
def test_resnet50_vs_torchvision():
    tv = pytest.importorskip("torchvision")
    spec, x = build_model("resnet50")
    env = om.run_model(spec, x)
    m = tv.models.resnet50().double().eval()
    convs = [l for l in spec["layers"] if l["op"] == "conv"]
    it = iter(convs)
    _set_conv(m.conv1, m.bn1, next(it))
    for stage in (m.layer1, m.layer2, m.layer3, m.layer4):
        for bi, blk in enumerate(stage):
            _set_conv(blk.conv1, blk.bn1, next(it))
            _set_conv(blk.conv2, blk.bn2, next(it))
            if bi == 0:
                _set_conv(blk.downsample[0], blk.downsample[1], next(it))
            _set_conv(blk.conv3, blk.bn3, next(it))
    fc = [l for l in spec["layers"] if l["op"] == "linear"][0]
    m.fc.weight.data = torch.from_numpy(fc["w"].astype(np.float64))
    m.fc.bias.data = torch.from_numpy(fc["b"].astype(np.float64))
    from oracle.ops import bf16_rne
    with torch.no_grad():
        logits = m(torch.from_numpy(bf16_rne(x)))
    ref = torch.softmax(logits, -1).numpy()
    assert _rel(env[spec["outputs"][0]], ref) < 1e-9
    # the logits too (softmax can hide errors)
    assert _rel(env[fc["out"]], logits.numpy()) < 1e-10


@pytest.mark.slow
def test_mobilenet_v2_vs_torchvision():
    tv = pytest.importorskip("torchvision")
    spec, x = build_model("mobilenet_v2")
    env = om.run_model(spec, x)
    m = tv.models.mobilenet_v2().double().eval()
    convs = iter([l for l in spec["layers"] if l["op"] == "conv"])
    f = m.features
    _set_conv(f[0][0], f[0][1], next(convs))
    for blk in f[1:18]:
        seq = list(blk.conv)
        # [ConvBNAct(expand)?], ConvBNAct(dw), Conv2d(project), BN
        for mod in seq[:-2]:
            _set_conv(mod[0], mod[1], next(convs))
        _set_conv(seq[-2], seq[-1], next(convs))
    _set_conv(f[18][0], f[18][1], next(convs))
    fc = [l for l in spec["layers"] if l["op"] == "linear"][0]
    m.classifier[1].weight.data = torch.from_numpy(fc["w"].astype(np.float64))
    m.classifier[1].bias.data = torch.from_numpy(fc["b"].astype(np.float64))
    from oracle.ops import bf16_rne
    with torch.no_grad():
        logits = m(torch.from_numpy(bf16_rne(x)))
    assert _rel(env[fc["out"]], logits.numpy()) < 1e-10
    assert _rel(env[spec["outputs"][0]], torch.softmax(logits, -1).numpy()) < 1e-10


@pytest.mark.slow
def test_bert_base_vs_hf():
    tr = pytest.importorskip("transformers")
    spec, x = build_model("bert_base")
    env = om.run_model(spec, x)
    cfg = tr.BertConfig(hidden_act="gelu", layer_norm_eps=1e-12, hidden_dropout_prob=0.0,
                        attention_probs_dropout_prob=0.0)
    m = tr.BertModel(cfg, add_pooling_layer=True).double().eval()
    L = spec["layers"]
    T = lambda a: torch.from_numpy(np.asarray(a, dtype=np.float64))  # noqa: E731
    emb = m.embeddings
    emb.position_embeddings.weight.data.zero_()
    emb.token_type_embeddings.weight.data.zero_()
    emb.LayerNorm.weight.data = T(L[0]["gamma"])
    emb.LayerNorm.bias.data = T(L[0]["beta"])
    emb.LayerNorm.eps = L[0]["eps"]
    idx = 1
    H = 768
    for layer in m.encoder.layer:
        qkv, qk, sm, pv, ao, ln1, f1, f2, ln2 = L[idx:idx + 9]
        idx += 9
        at = layer.attention
        for j, lin in enumerate((at.self.query, at.self.key, at.self.value)):
            lin.weight.data = T(qkv["w"][j * H:(j + 1) * H])
            lin.bias.data = T(qkv["b"][j * H:(j + 1) * H])
        at.output.dense.weight.data = T(ao["w"])
        at.output.dense.bias.data = T(ao["b"])
        at.output.LayerNorm.weight.data = T(ln1["gamma"])
        at.output.LayerNorm.bias.data = T(ln1["beta"])
        layer.intermediate.dense.weight.data = T(f1["w"])
        layer.intermediate.dense.bias.data = T(f1["b"])
        layer.output.dense.weight.data = T(f2["w"])
        layer.output.dense.bias.data = T(f2["b"])
        layer.output.LayerNorm.weight.data = T(ln2["gamma"])
        layer.output.LayerNorm.bias.data = T(ln2["beta"])
    pool = L[idx]
    m.pooler.dense.weight.data = T(pool["w"])
    m.pooler.dense.bias.data = T(pool["b"])
    with torch.no_grad():
        out = m(inputs_embeds=T(x)[None])
    assert _rel(env[spec["outputs"][0]], out.last_hidden_state[0].numpy()) < 1e-9
    assert _rel(env[spec["outputs"][1]], out.pooler_output.numpy()) < 1e-9


def test_model_flops_match_survey():
    """Algorithmic FLOPs per inference (48.4 M, 8.18 G, 0.602 G,
    22.35 G counting every GEMM incl. the 1-row pooler)."""
    got = {n: om.model_flops(build_model(n)[0]) for n in
           ("tiny_cnn", "resnet50", "mobilenet_v2")}
    assert got["tiny_cnn"] == pytest.approx(48.4e6, rel=0.01)
    assert got["resnet50"] == pytest.approx(8.18e9, rel=0.01)
    assert got["mobilenet_v2"] == pytest.approx(0.602e9, rel=0.01)
