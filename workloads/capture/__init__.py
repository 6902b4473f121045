"""Real-capture workload: a real PyTorch model captured
into a CUDA graph on the device, its allocation trace and kernel-node parameter
image, and the online-process emulation that rebuilds the graph from restored
parameters (see real_graph.py)."""
