#pragma once  // stand-in: tests/host/cuda_host_shim.h provides what the headers need
