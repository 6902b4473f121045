"""Offline / online phases of the real-capture check in separate processes
(SURVEY.md §8(f) NEXT-1, NEXT-2, NEXT-4).
  python tools/real_capture_online.py offline DIR   # capture + materialize, save
  python tools/real_capture_online.py online DIR    # fresh process: restore, rebuild, run
The online phase prints one JSON line."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_asplos_zengxgcl25_b200 as medusa  # noqa: E402
from workloads.capture import real_graph  # noqa: E402

phase, d = sys.argv[1], sys.argv[2]
os.makedirs(d, exist_ok=True)
if phase == "offline":
    print(json.dumps(real_graph.offline(torch, medusa, d)))
else:
    print(json.dumps(real_graph.online(torch, medusa, d)))
