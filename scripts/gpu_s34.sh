python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | tail -3
