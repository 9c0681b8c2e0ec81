"""The constants the paper prints (tests/golden/paper_constants.json) against what the code uses."""
import json
import os
import re

import idgsynth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G = json.load(open(os.path.join(ROOT, "tests", "golden", "paper_constants.json")))


def test_op_model():
    assert G["fma_in_phase"]["value"] + G["fma_in_accumulation"]["value"] == G["fma_per_sincos"]["value"]
    assert 2 * G["fma_per_sincos"]["value"] + 2 == G["ops_per_sincos_pair"]["value"]
    src = open(os.path.join(ROOT, "bench.py")).read()
    assert re.search(r"OPS_PER_PAIR\s*=\s*36\b", src)


def test_dataset_constants():
    assert len(idgsynth.baselines_for(G["ska1_low_stations"]["value"])) == G["ska1_low_baselines"]["value"]
    ska = idgsynth.CONFIGS["ska"]
    assert ska["T"] == G["timesteps"]["value"] and ska["slot"] == G["aterm_update_interval"]["value"]
    lofar = idgsynth.CONFIGS["lofar"]
    assert lofar["Ns"] == G["subgrid_size"]["value"] and lofar["N"] == G["grid_size"]["value"]
    assert lofar["C"] == G["channels"]["value"]
