"""Shared test/bench inputs: seeded synthetic images and pipeline descriptions.

Holds none of the method's arithmetic; see gen.py and pipelines.py headers."""
