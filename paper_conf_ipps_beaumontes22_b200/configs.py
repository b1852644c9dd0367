"""Load the BASELINE.json workloads from configs/*.json (written by
scripts/make_configs.py).  Pure data: no method arithmetic."""
from __future__ import annotations

import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CONFIG_DIR = os.path.join(ROOT, "configs")
NAMES = ["toy", "resnet50", "inception_v3", "vgg19", "gpt", "batch"]


def load(name: str) -> dict:
    with open(os.path.join(CONFIG_DIR, name + ".json")) as fh:
        return json.load(fh)
