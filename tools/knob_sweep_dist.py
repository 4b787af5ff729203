"""knob_sweep.py on another distribution -- dev tool: DIST FLAGS K"""
import sys, os
sys.argv = [sys.argv[0]] + sys.argv[2:] + [sys.argv[1]]
exec(open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "knob_sweep.py")).read()
     .replace('datagen.generate("uniform"', 'datagen.generate(sys.argv[3]'))
