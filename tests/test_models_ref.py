"""The oracle's model forwards (used for the CPU baseline and the reference
arm) run and produce the torchvision/HF output shapes; the cheap ones are
checked against an independent composition of the pinned layer oracle."""
import numpy as np

from oracle import layers_ref as L
from oracle import models_ref as M
from synth import tensors as syn


def test_tiny_models_match_layer_composition():
    y = M.mlp_forward(1000)
    g = syn.rng(1000)
    x = syn.activation(g, (256, 256)).astype(np.float64)
    for _ in range(3):
        w = syn.weight(g, (256, 256), 256).astype(np.float64)
        b = syn.bias(g, 256).astype(np.float64)
        x = np.maximum(x @ w.T + b, 0)
    assert np.allclose(y, x, rtol=1e-12, atol=1e-12)
    assert M.cnn_forward(1001).shape == (1, 32, 32, 16)


def test_model_output_shapes():
    assert M.mobilenet_v2_forward(1003).shape == (1, 1000)
    assert M.densenet121_forward(1002).shape == (1, 1000)
    y = M.bert_forward("base", 16, 1002)
    assert y.shape == (16, 768)
    assert np.allclose(y.mean(-1), 0, atol=0.6)   # post-LN rows (gamma ~ U(0.5,1.5), beta ~ N(0,0.1))
