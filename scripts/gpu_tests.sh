python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -5
timeout -s KILL 1200 python -m pytest tests -m gpu -q -x "$@" 2>&1 | tail -40
