from . import gen, configs  # noqa: F401
