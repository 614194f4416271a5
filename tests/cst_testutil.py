"""Shared helpers for the test-suite (imported as a plain module; tests/ is on sys.path)."""
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def gpu_available() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False
