"""Build a phase-timing variant of librtm (-DRTM_PHASE_TIMING) into /tmp and report cycles per tile phase."""
import ctypes, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
