"""Seeded synthetic inputs (no method arithmetic); see synth/workload.py."""
from .workload import *  # noqa: F401,F403
