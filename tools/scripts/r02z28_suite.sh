# full GPU suite + smoke on the current code
set -x
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
