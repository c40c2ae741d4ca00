"""Quick config-3 check (self-exchange, 512^3): V-cycle ms and exchange counts for k in {4, 8}, tb in {0, 1}."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from config_sweep import run  # noqa: E402

for k in (4, 8):
    for tb in (0, 1):
        run("c3", 512, 6, ghost_mode=1, transport=2, ca_period=[k] * 16, temporal_blocking=tb)
run("c3_noghost", 512, 6)
