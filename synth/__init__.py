"""Seeded synthetic inputs shared by tests, bench and both sides of parity checks.
Holds no arithmetic of the method (see configs.py / initial.py headers)."""
