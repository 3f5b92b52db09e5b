import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA (B200, sm_100a) device")
    config.addinivalue_line("markers", "slow: long-running")


# Measured parity errors, printed in the terminal summary of every run (also
# with -q): each GPU parity test calls record_err(name, err, detail).
_ERRS = []


def record_err(name, err, detail=""):
    _ERRS.append((name, float(err), str(detail)))


def pytest_terminal_summary(terminalreporter, exitstatus, config):
    if not _ERRS:
        return
    terminalreporter.write_sep("-", f"measured parity errors (max|err| / max|ref|), {len(_ERRS)} checks")
    for name, err, detail in _ERRS:
        terminalreporter.write_line(f"{err:10.3e}  {name}  {detail}")
