"""Shared pytest configuration.

Markers:
  gpu  — needs a CUDA device (B200); parity tests proper, calling through the C ABI.
Everything unmarked runs on CPU (oracle pins, host logic, ABI symbol export, gloo multi-process).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: test needs a CUDA GPU (B200)")
    config.addinivalue_line("markers", "slow: long-running test")
