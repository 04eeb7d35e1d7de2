"""Pins of the oracle's architecture tables against values printed in PAPER.md
(tests/golden/paper_pins.json, each with its citation) and shape invariants."""
import json
import os

import oracle

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_pins.json")))


def test_alexnet_721_725_mflops():
    # PAPER.md:219 §4.2.1: "partial CNN inference for fc7 (721 MFLOPS) independently of fc8 (725 MFLOPS)"
    fc7 = oracle.cnn_info(oracle.ALEXNET, 2)["macs_bias"]
    fc8 = oracle.cnn_info(oracle.ALEXNET, 3)["macs_bias"]
    assert round(fc7 / 1e6) == GOLD["alexnet_fc7_mflops"]["value"]
    assert round(fc8 / 1e6) == GOLD["alexnet_fc8_mflops"]["value"]
    # "incurring 99% redundant computations for fc8"
    assert int(100 * fc7 / fc8) == GOLD["alexnet_fc8_redundancy_pct"]["value"]


def test_resnet_784kb_layer():
    # PAPER.md:88 §1.1: one of ResNet50's layers is 784KB (fp32)
    i = oracle.cnn_info(oracle.RESNET50, 0)  # conv4_6
    assert (i["H"], i["W"], i["C"]) == (14, 14, 1024)
    assert i["act"] * 4 == GOLD["resnet50_layer_kb"]["value"] * 1024


def test_resnet_conv5_over_400000():
    # PAPER.md:185 §4.1: "conv5 of ResNet has over 400,000 features" (bytes, reading R25)
    for t in (1, 2, 3):
        i = oracle.cnn_info(oracle.RESNET50, t)
        assert (i["H"], i["W"], i["C"]) == (7, 7, 2048)
        assert i["act"] * 4 > GOLD["resnet50_conv5_features_over"]["value"]
        assert i["act"] * 4 == 401408


def test_alexnet_fc6_4096():
    assert oracle.cnn_info(oracle.ALEXNET, 1)["d"] == GOLD["alexnet_fc6_features"]["value"]


def test_top_tap_is_1000_wide():
    # PAPER.md:708-711 Table 2: top layer 0.08 GB for 20k rows in all three CNNs
    g = GOLD["top_layer_gb_foods"]
    for cnn in (oracle.ALEXNET, oracle.VGG16, oracle.RESNET50):
        t = oracle.n_taps(cnn) - 1
        d = oracle.cnn_info(cnn, t)["d"]
        assert round(g["n_rows"] * d * 4 / 1e9, 2) == g["value"]


def test_tap_widths_2x2_grid():
    # PAPER.md:369 fn 4: conv taps are max-pooled to a 2x2 grid of the same depth
    assert oracle.cnn_info(oracle.ALEXNET, 0)["d"] == 4 * 256
    assert oracle.cnn_info(oracle.RESNET50, 0)["d"] == 4 * 1024
    for t in (1, 2, 3):
        assert oracle.cnn_info(oracle.RESNET50, t)["d"] == 4 * 2048
    assert [oracle.cnn_info(oracle.VGG16, t)["d"] for t in range(3)] == [4096, 4096, 1000]


def test_mac_totals():
    # SURVEY.md §8a S1 (derived from the c.1 geometry): ResNet50 3862.2 M, VGG16 15572.2 M MACs/img
    assert round(oracle.cnn_info(oracle.RESNET50, 4)["macs"] / 1e5) == 38622
    assert round(oracle.cnn_info(oracle.VGG16, 2)["macs"] / 1e5) == 155722
    # fc6 input widths 9216 (AlexNet pool5 6x6x256) and 25088 (VGG pool5 7x7x512)
    a5, a6 = oracle.cnn_info(oracle.ALEXNET, 0)["macs"], oracle.cnn_info(oracle.ALEXNET, 1)["macs"]
    assert a6 - a5 == 9216 * 4096
    v6 = oracle.cnn_info(oracle.VGG16, 0)["macs"]
    v7 = oracle.cnn_info(oracle.VGG16, 1)["macs"]
    assert v7 - v6 == 4096 * 4096
